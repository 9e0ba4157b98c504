python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests -q -m gpu 2>&1 | tail -2
for W in 10000 3000000; do timeout 300 python tools/attn_exp.py --window $W 2>&1 | tail -1; done
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > /tmp/b.json 2>/tmp/b.err; python -c "import json;d=json.load(open('/tmp/b.json'));print(d['value'],d['ms_per_step'],d['roofline']['avg_launch_us'],d['stages_ms'])"
