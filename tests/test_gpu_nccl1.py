"""The NCCL wire of the multi-GPU path on the one
GPU a test box has: a 1-rank NCCL process group (in a fresh process, so the
group never outlives the test) runs every collective of parallel.py on CUDA
tensors -- blob broadcast (host-packed and device-built trees), in-place and
padded all-gathers, the max-over-ranks timer -- and the adopted tree's
traversal equals the original's.  Multi-rank flows are covered by the gloo
tests; this pins the NCCL calls themselves (device placement, dtypes,
in-place all_gather_into_tensor)."""
from __future__ import annotations

import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

_CHILD = r"""
import sys, numpy as np, torch, torch.distributed as dist
sys.path.insert(0, sys.argv[1])
import ttgen
import paper_conf_sc_goldfarbjk13_b200 as P
import paper_conf_sc_goldfarbjk13_b200.parallel as PAR
torch.cuda.set_device(0)
dist.init_process_group("nccl", device_id=torch.device("cuda", 0))
assert dist.get_backend() == "nccl"
dev = torch.device("cuda", 0)
b = ttgen.plummer(4096, seed=41)
bd = torch.from_numpy(b).cuda()
ref_tree = P.tt_tree_upload(P.build_oct(b))
ref = P.tt_traverse_bh(ref_tree, bd, 0.5, 0.05)
t1 = PAR.broadcast_tree(P.build_oct(b), dev)                    # host-packed blob over NCCL
t2 = PAR.broadcast_device_tree(P.tt_build_oct_device(bd), dev)  # device-built blob
for t in (t1, t2):
    assert torch.equal(P.tt_traverse_bh(t, bd, 0.5, 0.05), ref)
full = torch.arange(4096 * 4, dtype=torch.float32, device=dev).view(4096, 4)
keep = full.clone()
PAR.allgather_rows(full, 1)                                     # in-place all_gather_into_tensor
assert torch.equal(full, keep)
rng = PAR.balanced_ranges(torch.ones(4096, device=dev), 1)
PAR.allgather_rows_var(full, rng)
assert torch.equal(full, keep)
assert PAR.max_over_ranks(1.25, dev) == 1.25
torch.cuda.synchronize()
dist.destroy_process_group()
print("nccl ok")
"""


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.gpu
def test_nccl_collectives_one_rank():
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", MASTER_PORT=str(_free_port()), RANK="0", WORLD_SIZE="1",
               LOCAL_RANK="0")
    r = subprocess.run([sys.executable, "-c", _CHILD, ROOT], env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "nccl ok" in r.stdout, r.stdout + r.stderr
