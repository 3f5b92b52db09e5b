"""WinRS on B200 — fused Winograd backward-filter convolution (placeholder; binding lands with the C ABI)."""
