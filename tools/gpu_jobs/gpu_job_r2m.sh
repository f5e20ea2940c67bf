#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "partitioned or nccl or gs_inplace" > gpurun_out/r2m_tests.log 2>&1; echo pytest=$? >> gpurun_out/r2m_tests.log
timeout 600 python tools/dist_timing.py --configs 2 4 3 1 --out gpurun_out/r2m_dist.jsonl > gpurun_out/r2m_dist.log 2>&1
timeout 600 compute-sanitizer --tool memcheck python -c "
import torch, numpy as np, oracle, paper_conf_ipps_licqfsty16_b200 as sgr
from paper_conf_ipps_licqfsty16_b200 import gen
for g in (gen.stencil3d(12,11,10,27), gen.rmat(11,8,.57,.19,.19,seed=5)):
    rp=torch.from_numpy(g.row_ptr).cuda(); ci=torch.from_numpy(g.col_idx).cuda()
    for P in (2,3,8):
        r=sgr.color_partitioned(rp,ci,P); assert np.array_equal(r.colors.cpu().numpy(), oracle.jacobi(g,0).colors)
print('ok')
" > gpurun_out/r2m_memcheck.log 2>&1
