"""B200-native kernel fusion for image-processing pipelines (Qiao et al., CGO'19).

The product path: kfuse.Pipeline (C-ABI binding) -> libkfuse.so (planner,
code generator, NVRTC sm_100a kernels, executor).  No CPU fallback."""
from .kfuse import KfError, Pipeline, Plan, model_params, version  # noqa: F401
