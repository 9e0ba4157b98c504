# final session part 2: U1 bit-identity test, NEXT-2 / NEXT-3 / NEXT-1 / NEXT-4 measurements, parity error statistics
tag=$1; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -q -m gpu -k layer1_query > $out/u1test.log 2>&1; tail -2 $out/u1test.log
timeout 900 python tools/next2.py --out $out/next2.json 2>&1 | tail -4
timeout 900 python tools/next3.py --out $out/next3.json 2>&1 | tail -2
timeout 1500 python tools/sweep.py --out $out/sweep_L2k20.json > $out/sweep.log 2>&1; echo "sweep rc=$?"; tail -3 $out/sweep.log
timeout 1500 python tools/sweep.py --model 3,8 --out $out/sweep_L3k8.json > $out/sweep38.log 2>&1; echo "sweep38 rc=$?"; tail -3 $out/sweep38.log
timeout 1200 python tools/parity_errors.py --prec 0 1 4 2 3 --out $out/parity_errors.json 2>&1 | tail -6
