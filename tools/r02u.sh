python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
TG_GEMM_STG=-1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "gemm or embed_parity or f16x3" 2>&1 | tail -2
for d in 4 -1; do echo "STG=$d"; TG_GEMM_STG=$d python tools/gemm_bench.py --m 25000 --precs 1,4 --reps 10 2>&1 | grep -v "^$"; TG_GEMM_STG=$d python bench.py --no-cpu-baseline --no-profile --second-precision f16x3 > /tmp/b.json 2>/tmp/b.err; python -c "import json;d=json.load(open('/tmp/b.json'));print($d, d['value']/1e6, d['f16x3']['value']/1e6)" || tail -3 /tmp/b.err; done
