"""One diff-merge launch on 1 GiB streams (ncu target).

Usage: python scripts/merge_one.py [structure] [fraction]
  structure: suffix (default; the bench's case: the host owns the top of the buffer),
             scatter (Bernoulli, the worst case), runs (runs of 128 words)
  fraction:  share of the words the CPU changed (default 0.1)
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
import torch

from merge_bench import make
from paper_conf_cgo_panditg14_b200 import fcl

structure = sys.argv[1] if len(sys.argv) > 1 else "suffix"
frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.1
gpu, cpu, twin = make((1 << 30) // 4, frac, structure)
for _ in range(3):
    fcl.merge_raw(gpu.data_ptr(), cpu.data_ptr(), twin.data_ptr(), gpu.numel() * 4, 4,
                  torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize()
print("ok", structure, frac)
