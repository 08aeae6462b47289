# A/B of the fused-A paths on the skinny shape: TMA-staged (default) vs LDG converters
for st in 1 0; do echo "== A_STAGED $st"; EGEMM_A_STAGED=$st timeout 300 python tools/diag_skinny.py 2>&1 | grep -E "GEMM"; done
