python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for pp in 1 0 1 0; do
TG_PHI_PRE=$pp python bench.py --no-cpu-baseline --second-precision none > /tmp/b.json 2>/tmp/b.err; python -c "import json;d=json.load(open('/tmp/b.json'));k=d['roofline_kernels']['k_attn_g'];print('phi_pre', $pp, round(d['value']/1e6,3), 'attn us', round(k['avg_launch_us'],1), 'frac', round(k['frac'],3), d['stages_ms']['phi'])" || tail -3 /tmp/b.err
done
