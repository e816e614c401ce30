"""Seeded synthetic workloads (CSR on the host).  Holds no TileSpGEMM arithmetic."""
from .gen import CSR, config, CONFIGS  # noqa: F401
