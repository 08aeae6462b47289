#!/bin/bash
# Run every variant of tools/sanitize.py under compute-sanitizer's racecheck, synccheck and
# memcheck; one log per (tool, variant) under gpurun_out/sanitize/.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out/sanitize
VARS="${VARS:-presplit_256 presplit_224 presplit_128 presplit_128_sep cg1_128 cg1_128_sep fused_a_staged fused_a_ldg fused_a_128_sep fused_b presplit_256_s2 presplit_128_s3 presplit_256_ksplit3 cg1_128_ksplit2_sep fused_a_tail_peel tail_split fused_a_tail_split bf16_parts split knn_ar knn_stream knn_k64 knn_k32_stream knn_cg1 kmeans kmeans_e8 merge}"
for tool in ${TOOLS:-memcheck racecheck synccheck}; do
  for v in $VARS; do
    timeout 600 /usr/local/cuda/bin/compute-sanitizer --tool $tool --print-limit 20 \
      python tools/sanitize.py $v > gpurun_out/sanitize/${tool}_${v}.log 2>&1
    echo "$tool $v rc=$? $(tail -1 gpurun_out/sanitize/${tool}_${v}.log)"
  done
done
