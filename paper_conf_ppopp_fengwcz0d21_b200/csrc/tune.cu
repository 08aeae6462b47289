// tune.cu -- the measured tile / promotion / accumulator-mode table, which
// replaces the paper's analytic model (Sec. 6, Eqs. 2-8) by measurement.
//
// File: JSON written by tools/tune_sweep.py, read once (std::call_once) from
// $EGEMM_TUNE_TABLE or <dir of libegemm.so>/tune_table.json:
//   {"entries": [{"op": "gemm", "m_max": 128, "n_max": 1024, "k_max": 8192,
//                 "cg": 1, "bn": 128, "sep": 1, "kc": 256, "terms": 3, "stages": 3}, ...], ...}
// Value fields: cg, bn, sep, kc, fa (fused-split mask), terms (3 / 4; 0 = 3), stages (0 =
// the variant's default), n_slices (kNN; 0 = wave-balance formula), epi_warps (kMeans),
// ares (kNN query tile resident: -1 auto, 0 off).
// Lookup: the first entry (file order; the sweep writes them smallest bucket first) whose
// op matches and whose m_max/n_max/k_max bound (M, N, K).  Unknown keys are ignored.
// The parser accepts exactly this flat shape (objects of string/number fields inside the
// "entries" array) and rejects anything else by falling back to the built-in defaults.
#include <dlfcn.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>
#include "egemm_internal.h"

namespace egemm {

static std::vector<TuneEntry> g_table;
static std::string g_table_path;
static std::once_flag g_table_once;

static void skip_ws(const char*& p) {
  while (*p == ' ' || *p == '\n' || *p == '\r' || *p == '\t') p++;
}

static bool parse_string(const char*& p, std::string* out) {
  skip_ws(p);
  if (*p != '"') return false;
  p++;
  out->clear();
  while (*p && *p != '"') {
    if (*p == '\\' && p[1]) p++;
    out->push_back(*p++);
  }
  if (*p != '"') return false;
  p++;
  return true;
}

// skip any JSON value (used for fields we do not read)
static bool skip_value(const char*& p) {
  skip_ws(p);
  if (*p == '"') {
    std::string s;
    return parse_string(p, &s);
  }
  if (*p == '{' || *p == '[') {
    char open = *p, close = (*p == '{') ? '}' : ']';
    int depth = 0;
    bool in_str = false;
    for (; *p; p++) {
      if (in_str) {
        if (*p == '\\' && p[1]) p++;
        else if (*p == '"') in_str = false;
        continue;
      }
      if (*p == '"') in_str = true;
      else if (*p == open) depth++;
      else if (*p == close && --depth == 0) { p++; return true; }
    }
    return false;
  }
  char* end = nullptr;
  strtod(p, &end);
  if (end == p) {  // true / false / null
    if (!strncmp(p, "true", 4)) { p += 4; return true; }
    if (!strncmp(p, "false", 5)) { p += 5; return true; }
    if (!strncmp(p, "null", 4)) { p += 4; return true; }
    return false;
  }
  p = end;
  return true;
}

static bool parse_entry(const char*& p, TuneEntry* e) {
  skip_ws(p);
  if (*p != '{') return false;
  p++;
  for (;;) {
    skip_ws(p);
    if (*p == '}') { p++; return true; }
    std::string key;
    if (!parse_string(p, &key)) return false;
    skip_ws(p);
    if (*p != ':') return false;
    p++;
    skip_ws(p);
    if (key == "op") {
      std::string v;
      if (!parse_string(p, &v)) return false;
      e->op = v == "gemm" ? EPI_STORE : v == "knn" ? EPI_KNN : v == "kmeans" ? EPI_KMEANS
              : v == "gemm_b32" ? kOpGemmB32 : -1;
    } else if (key == "m_max" || key == "n_max" || key == "k_max" || key == "cg" || key == "bn" ||
               key == "sep" || key == "kc" || key == "fa" || key == "terms" || key == "stages" ||
               key == "n_slices" || key == "epi_warps" || key == "ares" || key == "peel" ||
               key == "ksplit" || key == "tsplit") {
      char* end = nullptr;
      long long v = strtoll(p, &end, 10);
      if (end == p) return false;
      p = end;
      if (key == "m_max") e->m_max = v;
      else if (key == "n_max") e->n_max = v;
      else if (key == "k_max") e->k_max = v;
      else if (key == "cg") e->cg = (int)v;
      else if (key == "bn") e->bn = (int)v;
      else if (key == "sep") e->sep = (int)v;
      else if (key == "fa") e->fa = (int)v;
      else if (key == "terms") e->terms = (int)v;
      else if (key == "stages") e->stages = (int)v;
      else if (key == "n_slices") e->nslices = (int)v;
      else if (key == "epi_warps") e->nepi = (int)v;
      else if (key == "ares") e->ares = (int)v;
      else if (key == "peel") e->peel = (int)v;
      else if (key == "ksplit") e->ksplit = (int)v;
      else if (key == "tsplit") e->tsplit = (int)v;
      else e->kc = (int)v;
    } else if (!skip_value(p)) {
      return false;
    }
    skip_ws(p);
    if (*p == ',') p++;
  }
}

static bool parse_table(const char* text, std::vector<TuneEntry>* out) {
  const char* p = strstr(text, "\"entries\"");
  if (!p) return false;
  p += 9;
  skip_ws(p);
  if (*p != ':') return false;
  p++;
  skip_ws(p);
  if (*p != '[') return false;
  p++;
  for (;;) {
    skip_ws(p);
    if (*p == ']') return true;
    TuneEntry e;
    if (!parse_entry(p, &e)) return false;
    if (e.op >= 0) out->push_back(e);
    skip_ws(p);
    if (*p == ',') p++;
  }
}

static void load_table() {
  std::string path;
  const char* env = getenv("EGEMM_TUNE_TABLE");
  if (env && *env) {
    path = env;
  } else {
    Dl_info info;
    if (dladdr(reinterpret_cast<void*>(&load_table), &info) && info.dli_fname) {
      std::string so = info.dli_fname;
      size_t slash = so.find_last_of('/');
      path = (slash == std::string::npos ? std::string(".") : so.substr(0, slash)) +
             "/tune_table.json";
    }
  }
  FILE* f = path.empty() ? nullptr : fopen(path.c_str(), "rb");
  if (!f) return;
  std::string text;
  char buf[4096];
  size_t n;
  while ((n = fread(buf, 1, sizeof(buf), f)) > 0) text.append(buf, n);
  fclose(f);
  std::vector<TuneEntry> t;
  if (parse_table(text.c_str(), &t)) {
    g_table.swap(t);
    g_table_path = path;
  }
}

bool tune_lookup(int op, long long M, long long N, long long K, TuneEntry* out) {
  std::call_once(g_table_once, load_table);
  for (const TuneEntry& e : g_table) {
    if (e.op != op || M > e.m_max || N > e.n_max || K > e.k_max) continue;
    *out = e;
    return true;
  }
  return false;
}

const char* tune_table_path() {
  std::call_once(g_table_once, load_table);
  return g_table_path.c_str();
}

int tune_table_size() {
  std::call_once(g_table_once, load_table);
  return (int)g_table.size();
}

}  // namespace egemm
