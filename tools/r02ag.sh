python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -2
for nk in "516 1032" "172 688"; do set -- $nk; echo "== N=$1 K=$2"; python tools/gemm_trace.py --n $1 --k $2 --precision tf32x3 --edges 60000 --mode 0 2>&1 | grep -E "landed"; done
python tools/gemm_bench.py --m 25000 --precs 1,4 --reps 10 2>&1 | grep -v "^$"
python bench.py --no-cpu-baseline --no-profile --second-precision f16x3 > /tmp/b.json 2>/tmp/b.err; python -c "import json;d=json.load(open('/tmp/b.json'));print(d['value']/1e6, d['f16x3']['value']/1e6)" || tail -3 /tmp/b.err
