cd $GRAFT_REPO_ROOT
O=gpurun_out/e8; mkdir -p $O
for i in 1 2; do
EGEMM_A_STAGED=0 timeout 300 python tools/shapes_time.py ldg >> $O/shapes.txt 2>&1
EGEMM_A_STAGED=0 EGEMM_A_PREFETCH=4 timeout 300 python tools/shapes_time.py ldg_pf4 >> $O/shapes.txt 2>&1
timeout 300 python tools/shapes_time.py staged >> $O/shapes.txt 2>&1
done
