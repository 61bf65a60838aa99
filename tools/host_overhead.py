"""Host cost of one ms_run call (the launch path: plan checks, tensor-map encode, occupancy query,
launch) vs its device time, for small inputs where a caller such as the delta-stepping loop issues
many calls back to back.  python tools/host_overhead.py [calls]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ppopp_ashkianidmo16_b200 import BucketSpec, Plan, _abi  # noqa: E402

calls = int(sys.argv[1]) if len(sys.argv) > 1 else 2000
L = _abi.lib()
for n, m, kv in ((1 << 12, 8, False), (1 << 16, 8, False), (1 << 20, 8, False), (1 << 16, 32, True),
                 (1 << 16, 256, False)):
    plan = Plan(BucketSpec.delta_range(m, (1 << 32) // m), n, with_values=kv)
    keys = torch.randint(0, 2**31, (n,), dtype=torch.int32, device="cuda")
    vals = keys.clone() if kv else None
    ko, vo = torch.empty_like(keys), (torch.empty_like(keys) if kv else None)
    off = torch.empty(m + 1, dtype=torch.int32, device="cuda")
    ws = plan.workspace(n)
    s = torch.cuda.current_stream().cuda_stream
    args = (plan._h, keys.data_ptr(), vals.data_ptr() if kv else None, None, ko.data_ptr(),
            vo.data_ptr() if kv else None, n, off.data_ptr(), ws.data_ptr(), ws.numel(), s)
    for _ in range(50):
        L.ms_run(*args)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record()
    for _ in range(calls):
        L.ms_run(*args)
    t_host = (time.perf_counter() - t0) / calls * 1e6
    e1.record()
    torch.cuda.synchronize()
    t_all = (time.perf_counter() - t0) / calls * 1e6
    t_dev = e0.elapsed_time(e1) / calls * 1e3
    print(f"n=2^{n.bit_length() - 1} m={m} {'KV' if kv else 'KO'}: host {t_host:6.2f} us/call (enqueue), "
          f"wall {t_all:6.2f} us/call, device stream {t_dev:6.2f} us/call, launches {plan.last_launches()}",
          flush=True)
