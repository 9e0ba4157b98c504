python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests -q -m gpu -x 2>&1 | tail -3
python tools/determinism.py lastfm 1
for c in lastfm reddit; do timeout 600 python bench.py --config $c --no-cpu-baseline --no-profile --second-precision none --steps 3 > /tmp/b.json 2>/tmp/b.err; python -c "import json;d=json.load(open('/tmp/b.json'));print('$c', round(d['value']/1e6,3))" || tail -3 /tmp/b.err; done
timeout 600 python tools/next3.py 2>&1 | tail -2
