"""B200-native GPL hot path (Paul, He, He, SIGMOD'16): fused, warp-specialised
scan -> filter -> hash-probe -> group-by pipeline for sm_100a behind a C ABI
(include/gpl.h, lib/libgpl.so). This package is the thin Python binding."""
from .gpl import Context, GplError, Result, load_library, merge_partials, version  # noqa: F401
