import numpy as np, torch, sys
sys.path.insert(0, '.')
from tests.gpu_helpers import setup, make_ctx
from tests.test_gpu_parity import _stream_gpu
from paper_conf_ppopp_wangm23_b200 import counters_dict, TG_NCOUNTERS
from tests.test_gpu_parity import _sim_counters
cfg, s, flat = setup("config1", n_edges=4000)
mc = cfg.model
want = _sim_counters(s, flat, mc, 700)
ref = None
bad = 0
for it in range(int(sys.argv[1])):
    for S in (1, 3, 16):
        ctx = make_ctx(s, flat, mc, cache_limit=700, superbatch=S)
        sc, log = _stream_gpu(ctx, s, mc.batch)
        ctx.close()
        simbad = [b for b, w in enumerate(want) if counters_dict(log[b], mc.n_layers) != w]
        if simbad:
            print("it", it, "S", S, "differs from the simulator at batches", simbad[:5], flush=True)
        if ref is None:
            ref = (sc, log); continue
        if not np.array_equal(log, ref[1]) or not np.array_equal(sc, ref[0]):
            bad += 1
            d = np.argwhere(log != ref[1])
            print("it", it, "S", S, "scores_eq", np.array_equal(sc, ref[0]), "diffs", d[:6].tolist(),
                  [(int(log[b, c]), int(ref[1][b, c])) for b, c in d[:6]])
print("bad", bad)
