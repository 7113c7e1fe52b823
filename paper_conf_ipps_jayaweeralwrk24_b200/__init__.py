"""DEFCON deformable-convolution inference hot path for NVIDIA B200 (sm_100a).

The compute lives in ``libdefcon.so`` (CUDA kernels behind the C ABI declared in
``include/defcon.h``); this package is the thin ctypes binding over it.  Build with
``python -m paper_conf_ipps_jayaweeralwrk24_b200.build``.
"""
from ._binding import (  # noqa: F401
    DefconError,
    TexPlan,
    defcon_abi_version,
    defcon_dcn_forward,
    defcon_deform_columns,
    defcon_dcn_workspace_size,
    defcon_layer_forward_host,
    defcon_layer_workspace_size,
    defcon_offset_dw_conv,
    defcon_offset_dw_conv_packed,
    defcon_offset_pack_params,
    defcon_offset_workspace_size,
    defcon_tex_filter_probe,
    load_library,
)
