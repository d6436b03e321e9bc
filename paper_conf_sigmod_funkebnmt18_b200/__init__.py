"""paper_conf_sigmod_funkebnmt18_b200 -- B200-native (sm_100a) HorseQC fused query pipelines.

libhq.so (csrc/, C ABI in include/hq.h) runs the hot path: hash builds, the
fused pipeline kernel (scan -> filter -> probe* -> aggregate | materialise),
finalisation and the operator-at-a-time baseline.  Python here is plumbing:
ctypes marshalling (hq), plan builders (engine, queries) and the multi-GPU
orchestration over torch.distributed / NCCL (dist).
"""
from . import hq  # noqa: F401
