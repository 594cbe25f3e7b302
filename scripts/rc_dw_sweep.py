"""Tuning build: C2 fused step at b = 8192 — whole step and dW-only device time (hb_bench_step) for
the current HB_RC_WGRAD_BN / HB_RC_WGRAD_S environment (one configuration per process)."""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_marws21_b200 as hb  # noqa: E402
from tests.helpers import dataset, init_params, params_to_flat, to_device  # noqa: E402

dims, b = [54, 512, 512, 512, 512, 7], 8192
m = hb.MLP(dims, precision="bf16")
m.set_params(params_to_flat(init_params(dims)))
w = hb.Worker(m, b)
X, y = dataset("covtype", b, seed=1)
tX, ty = to_device(X, y)
out = []
for part in (0, 2):
    us = C.c_float()
    rc = hb.lib.hb_bench_step(w.h, C.c_void_p(tX.data_ptr()), tX.stride(0), C.c_void_p(ty.data_ptr()), b, 50, part,
                              C.byref(us))
    out.append(f"part{part} {us.value:7.1f} us" if rc == 0 else f"part{part} error {hb.lib.hb_last_error()}")
print(f"BN={os.environ.get('HB_RC_WGRAD_BN', 'dflt')} S={os.environ.get('HB_RC_WGRAD_S', 'dflt')}:", "  ".join(out))
