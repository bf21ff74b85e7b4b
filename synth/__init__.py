"""Seeded synthetic inputs shared by the CPU oracle and the CUDA path.

This package holds NO arithmetic of the method (no model, loss, gradient,
merge or scaling).  It only draws the inputs the method consumes: the CSR
features and labels shaped like the paper's XML datasets (Table I,
PAPER.md P:1408-1413), the per-pass sample permutations, the initial model
parameters, and the per-config hyperparameters.  See DESIGN.md "Inputs".
"""
from .xmlgen import (CONFIGS, XmlConfig, Dataset, generate, init_params,
                     pass_permutation, sample_stream, config, param_layout,
                     planted_params)

__all__ = ["CONFIGS", "XmlConfig", "Dataset", "generate", "init_params",
           "pass_permutation", "sample_stream", "config", "param_layout", "planted_params"]
