"""B200-native ABFT Hessenberg reduction (Jia, Luszczek, Dongarra, IPDPSW 2016).

The product is libftgehrd.so (include/ftgehrd.h, CUDA for sm_100a); this
package is its thin Python binding.
"""
from .ftgehrd import (  # noqa: F401
    EV_NAMES, FT_E_UNCORRECTABLE, PHASE_AFTER_PANEL, PHASE_AFTER_RIGHT, PHASE_AFTER_UPDATE, PHASE_AT_END,
    PHASE_BEFORE_PANEL, POLICY_EAGER, POLICY_PAPER, SITE_A, SITE_C, SITE_K, SITE_R, SITE_CW, SITE_RW, SITE_T, SITE_V, SITE_Y, Report,
    build, dgehrd, dgehrd_host, dorghr, dsytrd, finalize, fortran, launch_count, lib, strerror, version,
    cyclic_columns, default_nb, dgehrd_mgpu, dgehrd_vranks, exchange_handles, global_to_local, mgpu_init,
    shard, unshard,
)
