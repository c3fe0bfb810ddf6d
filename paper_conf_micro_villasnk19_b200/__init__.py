"""nvbt — B200-native device-side instrumentation hot path of NVBit (Villa et al., MICRO'19).

`nvbt` is the ctypes binding of libnvbt.so (same names as include/nvbt.h); `drivers` holds the host
loops of the synthetic workloads (BFS level loop, stencil iterations, chunked replay) and the
multi-GPU merge. `build` compiles the library. Touching `nvbt` or `drivers` without the built library
raises ImportError: there is no fallback path.
"""
import importlib


def __getattr__(name):
    if name in ("nvbt", "drivers", "build"):
        return importlib.import_module(f".{name}", __name__)
    raise AttributeError(name)
