"""Seeded synthetic CSR input generators (no SpGEMM arithmetic). See synth/matrices.py."""
from .matrices import (Csr, values, from_coo, poisson2d, banded, webbase_like, qcd_like,
                       epidemiology_like, economics_like, circuit_like, rmat, random_sparse,
                       aggregation_prolongator, transpose,
                       MIXED, config)

__all__ = ["Csr", "values", "from_coo", "poisson2d", "banded", "webbase_like", "qcd_like",
           "epidemiology_like", "economics_like", "circuit_like", "rmat", "random_sparse", "aggregation_prolongator", "transpose",
           "MIXED", "config"]
