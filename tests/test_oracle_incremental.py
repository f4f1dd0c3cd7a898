"""The oracle's incremental evidence (batches of runs merged in ascending run order, used for the full-size
parity digests) equals the one-shot build on the same runs: it adds no arithmetic, only O4 applied batch by
batch."""
import pytest

import tracegen
from oracle import oracle


@pytest.mark.parametrize("cfg,div,nf,nr,batch", [(4, 128, 3, 5, 2), (9, 16, 4, 4, 3), (2, 64, 3, 3, 1), (5, 32, 2, 2, 4)])
def test_incremental_equals_one_shot(cfg, div, nf, nr, batch):
    p = tracegen.Params.preset(cfg, grid_div=div, runs_fix=nf, runs_rnd=nr)
    segs, _ = oracle.run_config(p)
    for cls in (0, 1):
        whole = oracle.build(segs[cls])
        ev = oracle.Evidence(cls)
        runs = sorted({s.run for s in segs[cls]})
        for k in range(0, len(runs), batch):
            ev.add([s for s in segs[cls] if s.run in runs[k:k + batch]])
        assert ev.export() == whole.export()


def test_incremental_rejects_out_of_order_runs():
    p = tracegen.Params.preset(1, runs_fix=3, runs_rnd=0)
    segs, _ = oracle.run_config(p)
    ev = oracle.Evidence(0)
    ev.add([s for s in segs[0] if s.run == 2])
    with pytest.raises(oracle.OracleError, match="ascending"):
        ev.add([s for s in segs[0] if s.run == 1])
