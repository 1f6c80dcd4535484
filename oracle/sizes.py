"""KV-cache size model (TEST INFRASTRUCTURE ONLY).

P:233 §3.3.2: KV cache per token = 2 x H x D x L x sizeof(FP16) bytes (H = KV heads,
D = head dim, L = layers); a user prefix of T_u tokens takes T_u x 2HDL x 2 bytes.
Table 2 P:396-403 prints the per-token figures for Qwen2-1.5B, Qwen2-7B and Llama3-1B.
"""

SIZEOF_FP16 = 2


def kv_bytes_per_token(kv_heads: int, head_dim: int, layers: int, elem_bytes: int = SIZEOF_FP16) -> int:
    return 2 * kv_heads * head_dim * layers * elem_bytes


def prefix_bytes(n_tokens: int, kv_heads: int, head_dim: int, layers: int) -> int:
    return n_tokens * kv_bytes_per_token(kv_heads, head_dim, layers)


def page_bytes(page_tokens: int, kv_heads: int, head_dim: int, layers: int) -> int:
    """One paged KV entry block holding page_tokens tokens of all layers."""
    return page_tokens * kv_bytes_per_token(kv_heads, head_dim, layers)
