mkdir -p gpurun_out/r02z
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python tools/parity_errors.py --prec 0 1 4 2 3 --out gpurun_out/r02z/parity_errors.json 2>&1 | tail -5
bash tools/sanitize.sh r02z
