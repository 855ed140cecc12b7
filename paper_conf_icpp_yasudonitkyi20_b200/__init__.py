"""B200-native Adaptive Bulk Search (Yasudo et al., ICPP 2020) hot path.

The product is libabs.so (C ABI in include/abs.h; kernels in csrc/).  This
package is its thin Python binding (abs.py) plus the in-tree build (build.py)
and the multi-GPU elite exchange (dist.py) over torch.distributed/NCCL."""
from .abs import (  # noqa: F401
    ABS_EEMPTY, ABS_EINVAL, ABS_OK, INIT_ALU, INIT_AUTO, INIT_MMA, MODE_ASYNC, MODE_LOCKSTEP, POLICY_SA, POLICY_WINDOW, AbsError, Solver, library_path, load,
    device_searches, ising_to_qubo, make_config, qubo_to_ising, random_qubo_dev, version, words,
)
