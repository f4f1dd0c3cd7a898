"""The N > 1 bench path end to end on one GPU (OWL_BENCH_SHARE_GPU=1: two ranks share cuda:0 over gloo): run
sharding, slot agreement, the owner exchange of the partial evidences (packed straight from the hash tables),
owner-side diff / KS tests and the library merge of the owners' rows (owl_merge_leaks / owl_merge_diffs) give
exactly the one-GPU oracle result over the same runs.  Config 9's launch sequences make
fix and rnd slot ids differ mid-sequence, so owner selection and the alignment-ordered merge are exercised."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import tracegen
from oracle import oracle

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

from tests.gpu_common import SIG, assert_leak_parity  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("cfg,runs", [(9, 6), (2, 2)])
def test_bench_two_ranks_equal_oracle(tmp_path, cfg, runs):
    env = dict(os.environ, OWL_BENCH_SHARE_GPU="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", "2", "--config", str(cfg), "--steps", "1",
           "--warmup", "1", "--no-cpu", "--no-e2e", "--runs", str(runs), "--dump", str(tmp_path)]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["n_gpus"] == 2 and line["config"]["parallelism"].startswith("dp2")
    meta = json.load(open(tmp_path / "runs.json"))
    p = tracegen.Params.preset(meta["config"], runs_fix=meta["runs_fix"], runs_rnd=meta["runs_rnd"])
    by_cls = {0: [], 1: []}
    for run in meta["runs"]:
        for m in tracegen.run_segments(p, run):
            by_cls[m.input_class].append(oracle.Segment(run, m.input_class, m.seq, m.n_warps, m.kernel_id,
                                                        tracegen.host_records(p, run, m.seq)))
    of, orr = oracle.build(by_cls[0]), oracle.build(by_cls[1])
    assert_leak_parity(np.load(tmp_path / "leaks.npy"), oracle.leak_test(of, orr, SIG))
    gd, od = np.load(tmp_path / "diff.npy"), oracle.diff(of, orr)
    assert len(gd) == len(od) and np.array_equal(gd, od)
