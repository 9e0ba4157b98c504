python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "embed_parity or time_encode or stream_bench_config or fp32_level or counters" 2>&1 | tail -2
for v in 1 0 1; do TG_PHI_TABLE=$v python bench.py --no-cpu-baseline --second-precision none > /tmp/b.json 2>/tmp/b.err; python -c "import json;d=json.load(open('/tmp/b.json'));k=d['roofline_kernels']['k_attn_g'];print('phi_table', $v, round(d['value']/1e6,3), 'attn us', round(k['avg_launch_us'],1), 'frac', round(k['frac'],3), d['stages_ms']['phi'], d['stats']['time_table_hit_rate'])" || tail -3 /tmp/b.err; done
python tools/determinism.py reddit 1
