python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for gr in 148 74 37; do echo "== grid $gr"; TG_GEMM_GRID=$gr python tools/gemm_trace.py --n 516 --k 1032 --precision tf32x3 --edges 60000 --mode 0 2>&1 | grep -E "landed"; TG_GEMM_GRID=$gr python tools/gemm_bench.py --m 25000 --precs 1 --reps 5 2>&1 | grep "516"; done
