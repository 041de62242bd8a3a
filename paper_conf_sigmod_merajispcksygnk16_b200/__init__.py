"""paper_conf_sigmod_merajispcksygnk16_b200 — B200-native hash GROUP BY (libblugby) after
Meraji et al., SIGMOD'16. The product is the C-ABI library libblugby.so (include/blu_gby.h);
`blugby` is its thin Python binding and `dist` the multi-GPU (torch.distributed / NCCL) layer."""
from . import blugby  # noqa: F401  (raises ImportError if libblugby.so is not built)
from .blugby import *  # noqa: F401,F403
