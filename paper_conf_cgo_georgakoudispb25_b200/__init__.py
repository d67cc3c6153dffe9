"""paper_conf_cgo_georgakoudispb25_b200 -- B200-native runtime kernel specialization.

A from-scratch implementation of the data-parallel hot path of Proteus (Georgakoudis,
Parasyris, Beckingsale, CGO '25): GPU kernels specialized at launch time on annotated
scalar arguments and launch dimensions, compiled once per specialization with NVRTC for
sm_100a, cached in memory and on disk, and dispatched with cuLaunchKernel.

  proteus.py    ctypes binding of libproteus.so (C ABI: include/proteus.h)
  workloads.py  the four workload kernels (Adam, 4th-order stencil, XS lookup,
                column microphysics) registered with libproteus + launch helpers
  halo.py       z-slab halo exchange for the multi-GPU stencil (torch.distributed)
  csrc/         libproteus C++ runtime and the CUDA kernel sources
"""
