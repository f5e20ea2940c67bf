"""paper_conf_ipps_licqfsty16_b200 — deterministic speculative-greedy (SGR) graph coloring on B200.

Placeholder; the public API is filled in with the CUDA binding.
"""
