cd $GRAFT_REPO_ROOT
O=gpurun_out/final1; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit,temperature.gpu --format=csv > $O/smi.txt
timeout 1200 python -m pytest tests -m gpu -q > $O/gpu_tests.txt 2>&1; echo "rc=$?" >> $O/gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 > $O/bench20.json 2> $O/bench20.err
timeout 600 python bench.py --no-cpu > $O/bench200.json 2> $O/bench200.err
timeout 1800 bash tools/prof_all.sh r02 > $O/prof_all.log 2>&1
ls -la gpurun_out > $O/ls.txt
