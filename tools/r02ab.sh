python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for m in 0 1 2; do echo "== mode $m"; python tools/gemm_trace.py --n 516 --k 1032 --precision tf32x3 --edges 60000 --mode $m 2>&1 | grep -E "landed"; done
