"""One diff-merge launch on 1 GiB streams, 10 % of the words changed in runs of 128 (ncu target)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
import torch

from merge_bench import make
from paper_conf_cgo_panditg14_b200 import fcl

gpu, cpu, twin = make((1 << 30) // 4, 0.1, sys.argv[1] if len(sys.argv) > 1 else "runs")
for _ in range(3):
    fcl.merge_raw(gpu.data_ptr(), cpu.data_ptr(), twin.data_ptr(), gpu.numel() * 4, 4,
                  torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize()
print("ok")
