"""Full-size parity (BASELINE.json configs at their paper sizes, "100 fixed + 100 random" traces): the GPU
path through the C ABI against fixtures the CPU oracle wrote (tools/make_parity_digests.py, tests/golden/full_size/):
E_fix / E_rnd canonical dumps and the diff rows by SHA-256 (bit-exact), every KS row (K exact, D bit-identical,
p within 1e-9 relative) and every leak row.  C2 / C3 (44 GB) and C4 (134 GB) are built in one fold launch per
class, the bench's launch configuration; C5 (184 GB, more than one B200 holds) in two chunks of runs merged with
owl_adcfg_accumulate."""
import hashlib
import json
import os

import numpy as np
import pytest

import tracegen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

from paper_conf_dsn_zhaoxcqzj24_b200 import api  # noqa: E402
from tests.gpu_common import SIG, assert_ks_parity, assert_leak_parity  # noqa: E402

GOLD = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "full_size")
CHUNK_BYTES = 140e9  # records resident at once (B200: 180 GB HBM)


def _fixture(cfg):
    path = os.path.join(GOLD, f"C{cfg}.json")
    if not os.path.exists(path):
        pytest.skip(f"no oracle fixture {path} (tools/make_parity_digests.py)")
    with open(path) as f:
        doc = json.load(f)
    z = np.load(os.path.join(GOLD, f"C{cfg}.npz"))
    return doc, z["ks"], z["leaks"]


def _chunks(p):
    runs = list(range(p.n_runs))
    per_run = 16 * sum(tracegen.host_count(p, r, m.seq) for r in runs[:2] for m in tracegen.run_segments(p, r)) / 2
    k = max(2, int(CHUNK_BYTES // max(per_run, 1)))
    return [runs[i:i + k] for i in range(0, len(runs), k)]


def _build_full(ctx, p, channel_order=False):
    ev = {0: None, 1: None}
    n_rec = 0
    for chunk in _chunks(p):
        segs = []
        for r in chunk:
            for m in tracegen.run_segments(p, r):
                buf, n = tracegen.device_records(p, r, m.seq)
                if channel_order:
                    buf = tracegen.device_interleave(buf, n)
                segs.append(api.Segment(r, m.input_class, m.seq, m.n_warps, m.kernel_id, buf, n,
                                        flags=0 if channel_order else api.OWL_SEG_WARP_MAJOR))
                n_rec += n
        torch.cuda.synchronize()
        ctx.ingest(segs)
        try:
            for c in (0, 1):
                rc = [r for r in chunk if tracegen.run_class(p, r) == c]
                if not rc:
                    continue
                if ev[c] is None:
                    ev[c] = ctx.build(rc)
                else:
                    ev[c].accumulate(rc)
        finally:
            ctx.forget_runs(chunk)
            del segs
            torch.cuda.empty_cache()
    return ev[0], ev[1], n_rec


@pytest.mark.parametrize("cfg,channel_order", [(1, False), (2, False), (3, False), (4, False), (5, False), (2, True),
                                               (2, "inplace")])
def test_full_size_parity(cfg, channel_order):
    """(2, True): the bench's workload in a tracer channel's order (bursts of 32, warps round-robin) gives the
    same A-DCFGs (reading R17), through the burst bucketing with the bursts copied to warp-major order;
    (2, "inplace"): the same, folded in place through the burst index (owl_config.channel_order, the default)."""
    doc, o_ks, o_leaks = _fixture(cfg)
    p = tracegen.Params.preset(cfg)
    assert (p.runs_fix, p.runs_rnd) == (doc["runs_fix"], doc["runs_rnd"])
    ctx = api.Context(0)
    if channel_order:
        ctx.set_config(channel_order=api.OWL_CHANNEL_IN_PLACE if channel_order == "inplace" else api.OWL_CHANNEL_COPY)
    ef, er, n_rec = _build_full(ctx, p, bool(channel_order))
    assert n_rec == doc["records"]
    bf, br = ef.export(), er.export()
    assert (len(bf), len(br)) == (doc["e_fix_bytes"], doc["e_rnd_bytes"])
    assert hashlib.sha256(bf).hexdigest() == doc["e_fix_sha256"], "E_fix differs from the oracle"
    assert hashlib.sha256(br).hexdigest() == doc["e_rnd_sha256"], "E_rnd differs from the oracle"
    d = ctx.diff(ef, er)
    assert len(d) == doc["diff_rows"] and hashlib.sha256(d.tobytes()).hexdigest() == doc["diff_sha256"]
    assert_ks_parity(ctx.ks_tests(ef, er, SIG), o_ks)
    assert_leak_parity(ctx.leak_test(ef, er, SIG), o_leaks)
