"""B200-native PGAS-style EMB-layer forward (Chen, Buluc, Yelick, Owens, SC 2024).

libemb.so (csrc/, C ABI in include/emb.h) holds every kernel; `emb` is the thin
binding with the same names; `layer.PgasEmbedding` is the rank-level convenience
object; `comm` builds the one-time IPC-handle all-gather.
"""
__version__ = "0.1.0"
