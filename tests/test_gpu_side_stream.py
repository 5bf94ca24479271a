"""GPU parity of the a2 / a3 side-stream section (csrc/igd.cu SideSection): the sync sort, epoch
tables and lock replay run on a second stream beside the a5 access sort when IGD_SIDE_STREAM=1
(by default only for lock-heavy traces).  The switch is read once per process, so each setting
runs in a child process; both must equal the CPU oracle on lock-heavy and lock-light traces,
single- and multi-tile, and on C2's sync-heavy variant."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
import tracegen as tg

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import json, sys
import numpy as np
sys.path.insert(0, sys.argv[1])
import paper_conf_sosp_kamathb21_b200 as igd
cases = json.loads(sys.argv[2])
out = {}
with igd.Detector(0) as d:
    for name, path, nb, bd in cases:
        ev = np.load(path)
        d.load(ev, nb, bd)
        d.detect()
        r = d.reports()
        np.save(path + ".gpu.npy", r)
print("ok")
"""


def _cases(tmp_path):
    import tracegen.families as F

    cases = []
    for seed, n, words, lock_words in [(61, 40_000, 30, 4), (62, 100_000, 3_000, 16), (63, 3_000, 5, 2)]:
        ev, nb, bd = tg.random_trace(seed, n, n_words=words,
                                     weights=[12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1], lock_words=lock_words,
                                     p_lock_data=0.2)
        cases.append((f"locks{seed}", ev, nb, bd))
    ev, nb, bd = tg.random_trace(64, 60_000, n_words=500)  # lock-light
    cases.append(("light64", ev, nb, bd))
    plan = F.Plan(2, 2_000_000, **F.SYNC_HEAVY)
    cases.append(("c2_sync_heavy", plan.fill(), plan.n_blocks, plan.block_dim))
    plan.close()
    out = []
    for name, ev, nb, bd in cases:
        p = str(tmp_path / f"{name}.npy")
        np.save(p, ev)
        out.append((name, p, int(nb), int(bd), ev))
    return out


@pytest.mark.parametrize("side", ["1", "0"])
def test_side_stream_vs_oracle(tmp_path, side):
    cases = _cases(tmp_path)
    env = dict(os.environ, IGD_SIDE_STREAM=side)
    arg = json.dumps([(c[0], c[1], c[2], c[3]) for c in cases])
    r = subprocess.run([sys.executable, "-c", CHILD, ROOT, arg], env=env, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    for name, p, nb, bd, ev in cases:
        got = np.load(p + ".gpu.npy")
        want = oracle.run(ev, nb, bd)
        assert len(got) == len(want), f"{name} side={side}: {len(got)} vs {len(want)}"
        assert np.array_equal(got, want), f"{name} side={side}"
