#!/bin/bash
# Round profiling pass (run on the GPU box from the repo root):  bash tools/prof_all.sh r02
# ncu --set full of the bench's kernels (one launch each) + the bench's launch list, and the
# bench's traffic source profiles/ncu_summary.json (identified by config and shape).
set -x
R=${1:-r02}
O=gpurun_out
NCU="ncu --set full --clock-control none --import-source on"
cfg5=$(python -c "from paper_conf_ppopp_fengwcz0d21_b200 import egemm; print(*egemm.query_config('gemm', 8192, 8192, 8192, with_fused=True))")
timeout 600 $NCU -k regex:egemm_tc_kernel -c 1 -f -o $O/${R}_gemm8192 python tools/prof_gemm.py 8192 2 > $O/ncu_gemm.log 2>&1
timeout 300 $NCU -k regex:split -c 2 -f -o $O/${R}_split python tools/prof_gemm.py 8192 1 > $O/ncu_split.log 2>&1
timeout 600 $NCU -k regex:egemm_tc_kernel -c 1 -f -o $O/${R}_knn python tools/prof_apps.py knn > $O/ncu_knn.log 2>&1
timeout 600 $NCU -k regex:"egemm_tc_kernel|km_" -c 10 -f -o $O/${R}_kmeans python tools/prof_apps.py kmeans > $O/ncu_kmeans.log 2>&1
timeout 600 $NCU -k regex:egemm_tc_kernel -c 1 -f -o $O/${R}_skinny python tools/prof_skinny.py > $O/ncu_skinny.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file $O/${R}_bench_launches.csv python bench.py --steps 2 --warmup 3 > $O/ncu_bench.log 2>&1
python tools/ncu_summarize.py $O/${R}_ncu $O/${R}_gemm8192.ncu-rep $O/${R}_split.ncu-rep \
  $O/${R}_knn.ncu-rep $O/${R}_kmeans.ncu-rep $O/${R}_skinny.ncu-rep --launch $O/${R}_bench_launches.csv --headline 15
python tools/ncu_summarize.py --bench-summary profiles/ncu_summary.json "$cfg5" "8192 8192 8192" \
  $O/${R}_gemm8192.ncu-rep $O/${R}_split.ncu-rep "profiles/${R}_ncu.md"
ls -la $O
