python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
TG_TRACE=1 python -m paper_conf_ppopp_wangm23_b200.build > /dev/null 2>&1
for p in tf32x3 f16x3; do for nk in "516 1032" "172 688" "1032 172"; do set -- $nk; echo "== $p N=$1 K=$2"; python tools/gemm_trace.py --n $1 --k $2 --precision $p --edges 60000 2>&1 | tail -14; done; done
