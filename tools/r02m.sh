python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for d in 4 1 0; do echo "== STG=$d"; TG_GEMM_STG=$d python tools/gemm_trace.py --n 172 --k 688 --precision tf32x3 --edges 60000 2>&1 | grep -E "landed|mma_commit"; TG_GEMM_STG=$d python tools/gemm_bench.py --m 25000 --precs 1,4 --reps 10 2>&1 | grep -v "^$"; done
