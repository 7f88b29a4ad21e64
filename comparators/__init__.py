"""Comparators (not the product path): the paper's own design in torch/cuBLAS."""
