"""The cross-GPU merge through a real NCCL process
group on the B200: world size 1 (gpurun gives one GPU), so the packed
all-gather of the padded front runs as an NCCL kernel, and the merged front
must equal the local one and the oracle's."""
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from magis_inputs import CandidateGenerator, CandidateSpec, build_workload  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph, pareto_merge  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import distributed as pdist  # noqa: E402


def test_nccl_global_front_world1():
    import torch.distributed as dist
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1, device_id=dev)
    try:
        assert dist.get_backend() == "nccl"
        wl = build_workload("c2")
        K = 4096
        P, D = CandidateGenerator(wl, CandidateSpec(seed=3)).generate(0, K)
        g = Graph.from_workload(wl)
        st, pk, lt = g.eval_schedules(torch.from_numpy(P).to(dev), torch.from_numpy(D).to(dev))
        cap = 1024
        M = int(wl.size.sum() // 8)
        local = pareto_merge(pk, lt, st, cap=cap, mem_limit=M)
        glob = pdist.global_front(local, cap, mem_limit=M)
        torch.cuda.synchronize()
        n = int(local["front_n"].item())
        assert int(glob["front_n"].item()) == n
        assert torch.equal(glob["front_id"][:n], local["front_id"][:n])
        assert torch.equal(glob["best"][:1], local["best"][:1])
        ref = oracle.pareto(pk.cpu().numpy(), lt.cpu().numpy(), st.cpu().numpy())
        assert np.array_equal(glob["front_id"][:n].cpu().numpy(), ref)
    finally:
        dist.destroy_process_group()
