"""paper_conf_cluster_chukzsp20_b200 -- B200-native dynamic kernel fusion for bulk
non-contiguous (MPI derived datatype) pack / unpack and halo exchange.

Thin ctypes binding over ``libddt.so`` (the C ABI in ``include/ddt.h``): every
call below only marshals arguments; every byte of the hot path is moved by the
library's sm_100a kernels.  There is no CPU fallback: if ``libddt.so`` is
missing, importing the binding raises (build it with
``python -m paper_conf_cluster_chukzsp20_b200.build`` or ``__graft_entry__.build()``).

PyTorch is used only for device memory (tensors' ``data_ptr``), streams
(``torch.cuda.current_stream().cuda_stream``) and process groups (to broadcast
the NCCL unique id and CUDA-IPC window handles).

Names follow the paper (Chu et al., PAPER.md): requests are enqueued into the
request list and launched by ``flush`` as one fused kernel (§IV-A);
``Halo`` is the bulk halo exchange of Alg 3 / §IV-B.
"""
from __future__ import annotations

from ._abi import (DDTError, lib, check, LAYOUT_KINDS, BASE_CODES, STATE_NAMES,  # noqa: F401
                   DDT_XCHG_NCCL, DDT_XCHG_P2P, DDT_XCHG_P2P_DIRECT, DDT_PENDING, DDT_BUSY, DDT_COMPLETED)
from .types import Type  # noqa: F401
from .queue import Queue, Plan  # noqa: F401
from .halo import Halo, Comm, Windows  # noqa: F401



def reload_env():
    """Make the library re-read its DDT_* experiment knobs (ddt_reload_env):
    call after changing one of those environment variables at run time."""
    lib().ddt_reload_env()


__all__ = ["reload_env", "DDTError", "Type", "Queue", "Plan", "Halo", "Comm", "Windows", "lib", "DDT_XCHG_NCCL", "DDT_XCHG_P2P"]
