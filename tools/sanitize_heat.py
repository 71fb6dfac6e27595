"""compute-sanitizer target: heat sweeps only (odd and even widths), each grid
in its own exact-size cudaMalloc (run with PYTORCH_NO_CUDA_MEMORY_CACHING=1) so
memcheck sees any read past the end of T1."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ppopp_xutycc14_b200 as xr  # noqa: E402

for nj, ni in [(33, 67), (9, 5), (41, 1027), (7, 2049), (20, 514)]:
    T0 = oracle.heat_init(nj, ni)
    t1 = torch.from_numpy(T0).cuda()
    t2 = t1.clone()
    res = torch.zeros(3, dtype=torch.float64, device="cuda")
    assert xr.xr_heat_run(nj, ni, 3, t1.data_ptr(), t2.data_ptr(), res.data_ptr()) == 0
    torch.cuda.synchronize()
    assert res.cpu().tolist() == oracle.heat(nj, ni, 3, T0)[1].tolist(), (nj, ni)
print("sanitize heat OK")
