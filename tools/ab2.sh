# A/B: parity subset on the default build, then bench lines per variant
# usage: bash tools/ab2.sh <tag> [tests] -- variant specs "name:ENV=V:lib" (lib = variants/libtg_<lib>.so or empty)
out=gpurun_out/$1; shift; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" > $out/build.log 2>&1 || { tail $out/build.log; exit 1; }
if [ "$1" = tests ]; then shift
timeout 900 python -m pytest tests -m gpu -x -q -k "${TESTK:-embed or stream_scores or fullsize_reddit or superbatch_invariance or opts_invariance or score_pairs or counters}" > $out/tests.log 2>&1; tail -3 $out/tests.log
fi
for spec in "$@"; do
  IFS=: read name envs lib <<< "$spec"
  for rep in 1 2; do
    l=""; [ -n "$lib" ] && l=variants/libtg_$lib.so
    env $envs TG_LIB=$l timeout 600 python bench.py --steps 5 --warmup 3 --second-precision ${PREC2:-none} --no-cpu-baseline > $out/bench_${name}_$rep.json 2> $out/bench_$name.err || tail -3 $out/bench_$name.err
    python - $out/bench_${name}_$rep.json $name <<'PY'
import json,sys
for l in open(sys.argv[1]):
    if l.startswith('{'):
        d=json.loads(l); k=d['roofline_kernels']; r=k['k_attn_g']
        g={n.split()[-1]:round(v['avg_launch_us'],1) for n,v in k.items() if 'gemm' in n}
        print(f"{sys.argv[2]:10s} value {d['value']/1e6:.3f} M  ms {d['ms_per_step']:.2f}  attn {r['avg_launch_us']:.1f} us frac {r['frac']:.3f} gemm {g}")
PY
  done
done
