"""Opt-in library modes, each in a fresh process (both are read once per
process): the L2 persisting window (TT_L2_PERSIST_MB) must not
change a result, and the bounds-checked build (TT_LIB=checked,
build.py --checked) must load and run the BH and kNN walks
trap-free with the product build's results."""
from __future__ import annotations

import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# one BH launch (child-group walk, 20k Plummer, theta 0.5) and one kNN launch,
# compared bit for bit with the same launches in the parent's product build
_CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import ttgen
import paper_conf_sc_goldfarbjk13_b200 as P
import paper_conf_sc_goldfarbjk13_b200._lib as L
b = ttgen.plummer(20000, seed=31)
tree = P.tt_tree_upload(P.build_oct(b))
bd = torch.from_numpy(b).cuda()
perm = P.tt_sort_points(tree, bd)
s = torch.cuda.Stream()
with torch.cuda.stream(s):  # a non-default stream: the window is a stream attribute
    acc = P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=perm)
torch.cuda.synchronize()
p = ttgen.gaussian_mixture(20000, 7, seed=32, components=12)
kt = P.tt_tree_upload(P.build_kd(p, 8))
idx, d2 = P.tt_traverse_knn(kt, torch.from_numpy(p[:5000]).cuda(), 8)
torch.cuda.synchronize()
np.savez(sys.argv[2], acc=acc.cpu().numpy(), idx=idx.cpu().numpy(), d2=d2.cpu().numpy(), lib=L.LIB_PATH)
"""


def _run(tmp_path, env_extra, tag):
    out = tmp_path / f"{tag}.npz"
    env = dict(os.environ, **env_extra)
    r = subprocess.run([sys.executable, "-c", _CHILD, ROOT, str(out)], env=env, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0, r.stdout + r.stderr
    import numpy as np
    return np.load(out), r.stderr


@pytest.mark.gpu
def test_l2_window_changes_no_result(tmp_path):
    import numpy as np
    base, _ = _run(tmp_path, {"TT_L2_PERSIST_MB": "0"}, "off")
    win, err = _run(tmp_path, {"TT_L2_PERSIST_MB": "64"}, "on")
    assert "L2 persisting window set" in err, err  # the window was really applied
    for k in ("acc", "idx", "d2"):
        assert np.array_equal(base[k], win[k]), k


@pytest.mark.gpu
def test_checked_build_runs_trap_free_with_product_results(tmp_path):
    import numpy as np
    lib = os.path.join(ROOT, "paper_conf_sc_goldfarbjk13_b200", "libtt_checked.so")
    if not os.path.exists(lib):
        pytest.skip("libtt_checked.so not built (build.py --checked)")
    base, _ = _run(tmp_path, {}, "product")
    chk, _ = _run(tmp_path, {"TT_LIB": "checked"}, "checked")
    assert str(chk["lib"]).endswith("libtt_checked.so")
    for k in ("acc", "idx", "d2"):
        assert np.array_equal(base[k], chk[k]), k
