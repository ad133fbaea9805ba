"""Embedding-layer integration: UGache as a drop-in torch module.

"UGache is wrapped into an embedding layer in PyTorch ... Applications can take advantage
of UGache's high-performance embedding extraction by replacing the reference of embedding
layer with UGache".  The table is read-only (pre-trained embeddings),
so the layer has no trainable parameters and its output does not require grad; the dense
model that consumes it trains as usual.  Marshalling only: rows are produced by
ugache_extract into a caller-visible [n, D] tensor of the table's element type.
"""
from __future__ import annotations

from typing import Optional

import torch

from .ugache import UGache


class UGacheEmbedding(torch.nn.Module):
    """``forward(keys) -> [*keys.shape, D]`` embedding rows of ``dtype`` on this GPU."""

    def __init__(self, cache: UGache, embedding_dim: int, dtype: torch.dtype = torch.float32):
        super().__init__()
        itemsize = torch.empty((), dtype=dtype).element_size()
        if embedding_dim * itemsize != cache.row_bytes:
            raise ValueError(f"D={embedding_dim} x {dtype} != row_bytes {cache.row_bytes}")
        self.cache = cache
        self.embedding_dim = embedding_dim
        self.dtype = dtype
        self._buf: Optional[torch.Tensor] = None

    def forward(self, keys: torch.Tensor, out: Optional[torch.Tensor] = None) -> torch.Tensor:
        flat = keys.reshape(-1)
        if flat.dtype not in (torch.int64, torch.int32):
            raise TypeError("keys must be int64 or int32")
        if not flat.is_contiguous():
            flat = flat.contiguous()
        n = flat.numel()
        if out is None:
            out = torch.empty((n, self.embedding_dim), dtype=self.dtype, device=keys.device)
        if out.dtype != self.dtype or out.numel() != n * self.embedding_dim or not out.is_contiguous():
            raise ValueError("out must be a contiguous [n, D] tensor of the layer dtype")
        self.cache.extract(flat, out, torch.cuda.current_stream(keys.device))
        return out.view(*keys.shape, self.embedding_dim)

    def extra_repr(self) -> str:
        return f"rows={self.cache.num_rows}, dim={self.embedding_dim}, dtype={self.dtype}"
