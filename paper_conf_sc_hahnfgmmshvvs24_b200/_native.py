"""ctypes loader for libmdnorm.so (argument marshalling only; no compute happens here).

The library is required: a missing or unloadable library raises immediately at first use -- there
is no CPU fallback anywhere in the product path.
"""
from __future__ import annotations

import ctypes as C
import os
import re

PKG = os.path.dirname(os.path.abspath(__file__))
# MDN_LIB_PATH: developer override to load an experimental build (tools/variants.sh)
LIB_PATH = os.environ.get("MDN_LIB_PATH") or os.path.join(PKG, "libmdnorm.so")
HEADER = os.path.join(os.path.dirname(PKG), "include", "mdnorm.h")

MDN_OK, MDN_EINVAL, MDN_ENOMEM, MDN_ECUDA, MDN_ESTATE = 0, 1, 2, 3, 4
MDN_ACC_F32, MDN_ACC_F64 = 0, 1
MDN_PRIV_AUTO, MDN_PRIV_OFF, MDN_PRIV_ON = -1, 0, 1
MDN_MAX_OPS, MDN_MAX_MATS = 48, 64
STATUS_NAMES = {0: "MDN_OK", 1: "MDN_EINVAL", 2: "MDN_ENOMEM", 3: "MDN_ECUDA", 4: "MDN_ESTATE"}

P, i64, i32, d = C.c_void_p, C.c_int64, C.c_int32, C.c_double

# name -> argtypes (restype is mdn_status = int unless listed in _RESTYPES)
SIGNATURES = {
    "mdnorm_create_grid": [C.c_int, P, P, P, P, C.c_int, P],
    "mdnorm_destroy": [P],
    "mdnorm_set_instrument": [P, i64, P, P],
    "mdnorm_set_flux": [P, i64, P, P],
    "mdnorm_accumulate": [P, P, P, i32, P, d, d, d, i64, i64, i64, P],
    "mdnorm_accumulate_runs": [P, P, i32, P, P, i32, P, d, d, i64, i64, i64, P],
    "binmd_accumulate": [P, P, i32, P, i64, P, i64, i32, i32, P],
    "mdnorm_histograms": [P, P, P, P],
    "mdnorm_cross_section": [P, P, P],
    "mdn_divide": [C.c_int, P, P, P, i64, P],
    "mdnorm_reset": [P, P],
    "mdnorm_set_pixel_krange": [P, i64, P, P],
    "mdnorm_set_flux_tables": [P, i32, P, P, P, i64, P],
    "binmd_accumulate_err": [P, P, i32, P, i64, P, i64, i32, i32, i32, P],
    "mdnorm_error_histogram": [P, P],
    "mdnorm_cross_section_err": [P, P, P, P],
    "mdnorm_stats": [P, C.c_int, P],
    "mdnorm_set_privatization": [P, i32],
    "mdnorm_accumulation_paths": [P, P],
    "mdn_last_error": [],
    "mdn_version": [],
    "mdnorm_accumulate_matrices": [P, i32, P, P, d, d, i64, i64, i64, P],
    "binmd_accumulate_matrices": [P, i32, P, i64, P, i64, i32, i32, P],
    "mdnorm_debug_trajectories": [P, i32, P, P, d, d, i64, P, P, P, P, P, i64],
    "binmd_debug_bins": [P, i32, P, i64, P, i64, i32, i32, P],
    "mdnorm_debug_compose": [P, P, i32, P, i32, P, P, P],
    "mdnorm_debug_set_max_slab": [P, i64],
    "mdnorm_debug_last_launch": [P, P],
    "mdnorm_debug_flux_guess": [P, i32, P],
    "binmd_box_bounds": [P, i64, P, i32, P, P],
    "binmd_accumulate_boxes": [P, P, i32, P, i64, P, i32, P, P],
}
_RESTYPES = {"mdn_last_error": C.c_char_p, "mdn_version": C.c_char_p}


class MdnError(RuntimeError):
    def __init__(self, status: int, where: str, msg: str):
        self.status = status
        super().__init__(f"{where}: {STATUS_NAMES.get(status, status)}: {msg}")


_lib = None


def header_functions() -> list[str]:
    """Names of every function declared in include/mdnorm.h."""
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return re.findall(r"^\s*(?:const\s+)?\w+\s*\*?\s*(\w+)\s*\(", src, flags=re.M)


def load() -> C.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(
                f"{LIB_PATH} is missing: build it with `python -m paper_conf_sc_hahnfgmmshvvs24_b200.build` "
                "(there is no CPU fallback)")
        lib = C.CDLL(LIB_PATH)
        dev_variant = "MDN_LIB_PATH" in os.environ  # tools/ A/B builds may predate newer debug entries
        for name, args in SIGNATURES.items():
            if dev_variant and not hasattr(lib, name):
                continue
            fn = getattr(lib, name)
            fn.argtypes = args
            fn.restype = _RESTYPES.get(name, C.c_int)
        _lib = lib
    return _lib


def check(status: int, where: str) -> None:
    if status != MDN_OK:
        raise MdnError(status, where, load().mdn_last_error().decode(errors="replace"))
