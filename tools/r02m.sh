python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for bn in 256 128; do for d in 4 2 1 0; do echo "BN=$bn STG=$d"; TG_X3_BN=$bn TG_GEMM_STG=$d python tools/gemm_bench.py --m 25000 --precs 1,4 --reps 10 2>&1 | grep -v "^$"; done; done
