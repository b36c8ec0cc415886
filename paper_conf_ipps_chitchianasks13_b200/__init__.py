"""B200-native distributed particle filter (Chitchian et al., IPDPS 2013).

The compute path is the C-ABI library ``libpf_b200.so`` (hand-written sm_100a
CUDA, sources in ``csrc/``); ``binding`` is its thin ctypes binding and
``ParticleFilter`` the torch-buffer front end.  Imports are lazy so that
``workload`` (the seeded input generator) can be used without the CUDA
library.
"""
import importlib

__all__ = ["ParticleFilter", "binding", "workload", "distributed"]


def __getattr__(name):
    if name == "ParticleFilter":
        return importlib.import_module(".filter", __name__).ParticleFilter
    if name in ("binding", "workload", "distributed"):
        return importlib.import_module("." + name, __name__)
    raise AttributeError(name)
