import time, ctypes, torch, numpy as np, sys
sys.path.insert(0, ".")
import tracegen
from paper_conf_dsn_zhaoxcqzj24_b200 import api, _lib
p = tracegen.Params.preset(2)
dev = torch.device("cuda", 0); stream = torch.cuda.current_stream(dev)
ctx = api.Context(0); segs = []
for r in range(40):
    for m in tracegen.run_segments(p, r):
        buf, n = tracegen.device_records(p, r, m.seq, device=dev, stream=stream)
        segs.append(api.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, buf, n))
torch.cuda.synchronize(); ctx.ingest(segs, stream)
rf = [r for r in range(40) if tracegen.run_class(p, r) == 0]; rr = [r for r in range(40) if tracegen.run_class(p, r) == 1]
for it in range(4):
    ef, er = ctx.build(rf), ctx.build(rr); torch.cuda.synchronize()
    t0 = time.perf_counter()
    pp, n = ctypes.c_void_p(), ctypes.c_size_t()
    st = _lib.load().owl_diff_adcfg(ctx.h, ef.h, er.h, ctypes.byref(pp), ctypes.byref(n))
    t1 = time.perf_counter()
    out = api._take(pp, n.value, api.DIFF_DTYPE)
    t2 = time.perf_counter()
    lk = ctx.leak_test(ef, er, 0.05)
    t3 = time.perf_counter()
    ef.destroy(); er.destroy()
    t4 = time.perf_counter()
    print(f"diff C {1e3*(t1-t0):.3f} ms, take {1e3*(t2-t1):.3f} ms, leak {1e3*(t3-t2):.3f} ms, destroy {1e3*(t4-t3):.3f} ms rows {n.value}")
