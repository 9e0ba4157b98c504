python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests -q -m gpu 2>&1 | tail -3
for W in 10000 3000000; do timeout 300 python tools/attn_exp.py --window $W 2>&1 | tail -1; done
