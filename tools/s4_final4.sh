# final build re-measurement: full GPU tests, smoke, bench, bench lines, NEXT-3, ncu launch list + full capture
tag=$1; out=gpurun_out/$tag; mkdir -p $out
bash tools/r02_full.sh $tag
bash tools/bench_all.sh $out
timeout 900 python tools/next3.py --out $out/next3.json 2>&1 | tail -2
bash tools/s4_final3.sh $tag tf32x3 2>&1 | grep -v "^memcheck\|^racecheck\|^synccheck"
