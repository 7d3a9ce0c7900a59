"""B200-native TBlock hot path of TGLite (Wang & Mendis, ASPLOS'24).

The compute path is libtgl.so (hand-written sm_100a CUDA behind include/tgl.h);
this package is its ctypes binding (`tgl`) and the host-side TBlock chain
(`block`).  Importing it fails loudly when libtgl.so has not been built: there is
no CPU fallback.
"""
from . import tgl  # noqa: F401  (raises ImportError if libtgl.so is missing)
from .block import HostStream, TBlock, TGATPipeline, TSampler  # noqa: F401

__all__ = ["tgl", "TBlock", "TGATPipeline", "TSampler", "HostStream"]
