"""B200-native retarded-potential step of Arumugam et al. (ICPP'17).

The product is the C-ABI library ``librp.so`` (``include/rp.h``, CUDA for sm_100a in
``csrc/``); ``rp`` is its thin ctypes binding and ``sim`` a small driver that strings the
four steps of the paper's loop together for one process / GPU, with
``torch.distributed`` plumbing for mesh-point sharding over ranks.
"""
__all__ = ["rp", "sim"]
