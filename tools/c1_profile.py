"""C1 epoch (2 virtual ranks, 1 MiB, block Pready g=16) for an ncu launch list."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
import torch
import paper_conf_sc_temucinslsga24_b200 as pc
from paper_conf_sc_temucinslsga24_b200 import apps
import bench
print(bench.c1_bench(pc, apps, torch, epochs=int(sys.argv[1]) if len(sys.argv) > 1 else 50))
