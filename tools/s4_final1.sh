# final session part 1: full GPU tests, smoke, bench (driver command), bench lines of every workload
tag=$1; out=gpurun_out/$tag; mkdir -p $out
bash tools/r02_full.sh $tag
bash tools/bench_all.sh $out
