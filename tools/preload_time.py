"""Time csmv_load_kv (the device KV preload) at C4's size: python -m tools.preload_time"""
import sys, time
import torch
sys.path.insert(0, ".")
from paper_conf_ipps_nunesc022_b200 import csmv

S, A, K = 1 << 22, 16, 4
with csmv.KvStore(S, A, K) as st:
    for i in range(5):
        torch.cuda.synchronize()
        t = time.perf_counter()
        st.load(S)
        print(f"load {i}: {1e3 * (time.perf_counter() - t):.2f} ms", flush=True)
