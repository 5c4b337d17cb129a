"""B200-native Eirene: batched, linearizable Query/Update/Insert/Delete processing
on a GPU-resident B+tree by combining (Zhang et al., PPoPP'23).

The product is the C-ABI library libeirene.so (include/eirene.h) built from
csrc/*.cu for sm_100a; this package holds the build script, the ctypes
binding, the torch-tensor wrapper (tree.EireneTree), the multi-GPU key-range
router (parallel.ShardedEirene) and the seeded workload generator.
"""
from . import workload  # noqa: F401

__all__ = ["workload", "EireneTree", "build"]


def __getattr__(name):
    if name == "EireneTree":
        from .tree import EireneTree
        return EireneTree
    if name == "build":
        from .build import build
        return build
    raise AttributeError(name)
