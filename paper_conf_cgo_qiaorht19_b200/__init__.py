"""B200-native kernel fusion for image-processing pipelines (Qiao et al., CGO'19).

The product path: kfuse.Pipeline (C-ABI binding) -> libkfuse.so (planner,
code generator, NVRTC sm_100a kernels, executor).  No CPU fallback.

The binding is imported lazily so that `paper_conf_cgo_qiaorht19_b200.build`
can run in a fresh tree before libkfuse.so exists; touching any exported name
without the library raises ImportError (fails loudly)."""

_EXPORTS = ("KfError", "Pipeline", "Plan", "model_params", "version")


def __getattr__(name):
    if name in _EXPORTS:
        from . import kfuse
        return getattr(kfuse, name)
    raise AttributeError(name)
