# A/B of library variants (variants/libtg_<name>.so) on the tf32x3 bench: per variant two bench
# runs (attention share + value), plus the default build; prints one line per run
out=gpurun_out/$1; shift; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail $out/build.log; exit 1; }
for v in default "$@"; do
  for rep in 1 2; do
    if [ $v = default ]; then lib=""; else lib=variants/libtg_$v.so; fi
    TG_LIB=$lib timeout 600 python bench.py --steps 5 --warmup 3 --second-precision none --no-cpu-baseline > $out/bench_${v}_$rep.json 2> $out/bench_$v.err
    python - $out/bench_${v}_$rep.json $v <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); r=d['roofline_kernels']['k_attn_g']
        print(f"{sys.argv[2]:10s} value {d['value']/1e6:.3f} M  ms {d['ms_per_step']:.2f}  attn {r['avg_launch_us']:.1f} us frac {r['frac']:.3f}")
PY
  done
done
