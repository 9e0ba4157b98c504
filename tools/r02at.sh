python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x 2>&1 | tail -2
for v in 1 2; do python bench.py --no-cpu-baseline --second-precision f16x3 > /tmp/b.json 2>/tmp/b.err; python -c "import json;d=json.load(open('/tmp/b.json'));k=d['roofline_kernels'];print(round(d['value']/1e6,3), round(d['f16x3']['value']/1e6,3), {n:round(v['avg_launch_us'],1) for n,v in k.items()})" || tail -3 /tmp/b.err; done
python tools/determinism.py reddit 1
