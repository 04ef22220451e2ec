"""pgvc — B200-native bounded instantiation of PUGpara's parameterized VCs.

Importing the package is cheap: the CUDA library is loaded on first use of the
binding (`paper_conf_ipps_lig12_b200.pgvc`).  `workloads` is pure input
definition and never touches the GPU.
"""
__all__ = ["workloads"]
