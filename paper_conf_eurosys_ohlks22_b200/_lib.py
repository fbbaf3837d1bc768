"""ctypes declarations of the C ABI in include/ooo.h (argument marshalling only).

Loading fails loudly if libooo.so has not been built: there is no fallback
path of any kind.
"""
from __future__ import annotations

import ctypes
import os
from ctypes import POINTER, c_char_p, c_double, c_float, c_int32, c_int64, c_size_t, c_void_p

LIB_PATH = os.environ.get("OOO_LIB") or os.path.join(os.path.dirname(os.path.abspath(__file__)), "lib",
                                                      "libooo.so")

OOO_OK = 0
STATUS = {0: "OOO_OK", 1: "OOO_ERR_INVALID_ARGUMENT", 2: "OOO_ERR_UNSUPPORTED", 3: "OOO_ERR_CUDA",
          4: "OOO_ERR_NCCL", 5: "OOO_ERR_STATE"}
DTYPES = {"bf16": 0, "fp32": 1}
ACTS = {"id": 0, "relu": 1, "gelu": 2}
SCHED_IN_ORDER = 0
SCHED_FIRST_K = 1
SCHED_REGIONS = 2
UNIQUE_ID_BYTES = 128


class StackDesc(ctypes.Structure):
    _fields_ = [
        ("num_layers", c_int32),
        ("dims", POINTER(c_int32)),
        ("acts", POINTER(c_int32)),
        ("tokens", c_int32),
        ("dtype", c_int32),
        ("need_input_grad", c_int32),
        ("bucket_layers", c_int32),
        ("max_temp_bytes", c_int64),
        ("W", POINTER(c_void_p)),
        ("b", POINTER(c_void_p)),
        ("grads", c_void_p),
        ("workspace", c_void_p),
        ("world_size", c_int32),
        ("rank", c_int32),
        ("nccl_unique_id", c_void_p),
        ("comm_enabled", c_int32),
        ("nccl_max_ctas", c_int32),
        ("wait_timeout_ms", c_int32),
        ("comm_priority", c_int32),
        ("comm_model_gbps", c_int32),
        ("comm_chunk_bytes", c_int64),
        ("average_over", c_int32),
        ("engine_ctas", c_int32),
    ]


class PipelineDesc(ctypes.Structure):
    _fields_ = [
        ("num_layers", c_int32),
        ("dims", POINTER(c_int32)),
        ("acts", POINTER(c_int32)),
        ("tokens", c_int32),
        ("group_layers", c_int32),
        ("n_stages", c_int32),
        ("placement", c_int32),
        ("W", POINTER(c_void_p)),
        ("b", POINTER(c_void_p)),
        ("workspace", c_void_p),
        ("grads", c_void_p),
        ("world_size", c_int32),
        ("rank", c_int32),
        ("nccl_unique_id", c_void_p),
    ]


class Schedule(ctypes.Structure):
    _fields_ = [("kind", c_int32), ("k", c_int32)]


class LaunchRecord(ctypes.Structure):
    _fields_ = [
        ("kind", c_int32),
        ("layer", c_int32),
        ("stream", c_int32),
        ("grid", c_int32),
        ("flops", c_double),
        ("bytes", c_double),
        ("ms", c_float),
        ("start_ms", c_float),
    ]


KIND_NAMES = {0: "fwd_gemm", 1: "dx_gemm", 2: "dw_gemm", 3: "seed", 4: "pack", 5: "allreduce", 6: "copy",
              7: "engine_fwd", 8: "engine_bwd", 9: "engine_step"}

EXPORTS = [
    "ooo_abi_version", "ooo_last_error", "ooo_status_string", "ooo_query_sizes", "ooo_grad_offsets",
    "ooo_schedule_order", "ooo_max_k", "ooo_deferral_bytes", "ooo_get_unique_id", "ooo_create_stack",
    "ooo_forward", "ooo_backward", "ooo_join", "ooo_graph_create", "ooo_graph_launch",
    "ooo_graph_destroy", "ooo_destroy", "ooo_tensor", "ooo_set_timing", "ooo_timing_read",
    "ooo_engine_plan", "ooo_region_schedule", "ooo_plan_regions", "ooo_region_plan", "ooo_k_search",
    "ooo_allreduce_buckets", "ooo_graph_set_timing_slots", "ooo_graph_timing_read", "ooo_comm_schedule",
    "ooo_comm_issue_order", "ooo_input_grad_wait", "ooo_pipeline_query_sizes", "ooo_pipeline_grads_offset",
    "ooo_pipeline_create", "ooo_pipeline_graph_create", "ooo_pipeline_stage_of", "ooo_pipeline_destroy",
    "ooo_graph_upload", "ooo_graph_launch_host",
]

_lib = None


class OooError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


def load() -> ctypes.CDLL:
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(
            f"{LIB_PATH} is missing: build it with `python -m paper_conf_eurosys_ohlks22_b200.build` "
            "(or __graft_entry__.build()); there is no fallback path")
    lib = ctypes.CDLL(LIB_PATH)
    S = c_int32
    lib.ooo_abi_version.restype = c_int32
    lib.ooo_last_error.restype = c_char_p
    lib.ooo_status_string.restype = c_char_p
    lib.ooo_status_string.argtypes = [c_int32]
    lib.ooo_query_sizes.restype = S
    lib.ooo_query_sizes.argtypes = [POINTER(StackDesc), POINTER(c_size_t), POINTER(c_size_t)]
    lib.ooo_grad_offsets.restype = S
    lib.ooo_grad_offsets.argtypes = [POINTER(StackDesc), POINTER(c_int64)]
    lib.ooo_schedule_order.restype = S
    lib.ooo_schedule_order.argtypes = [c_int32, Schedule, c_int32, POINTER(c_int32), POINTER(c_int32)]
    lib.ooo_max_k.restype = c_int32
    lib.ooo_max_k.argtypes = [c_int32, c_int64, POINTER(c_int64), POINTER(c_int64), c_int64]
    lib.ooo_deferral_bytes.restype = c_int64
    lib.ooo_deferral_bytes.argtypes = [POINTER(StackDesc), c_int32]
    lib.ooo_engine_plan.restype = S
    lib.ooo_engine_plan.argtypes = [POINTER(StackDesc), Schedule, c_int32, c_int32, POINTER(c_int32), c_int32,
                                    POINTER(c_int32), POINTER(c_int32)]
    lib.ooo_region_schedule.restype = S
    lib.ooo_region_schedule.argtypes = [c_int32, POINTER(c_double), c_int32, POINTER(c_double), POINTER(c_double),
                                        POINTER(c_double), POINTER(c_int32), POINTER(c_int64), c_int64,
                                        POINTER(c_int32), POINTER(c_int32), POINTER(c_int32)]
    lib.ooo_plan_regions.restype = S
    lib.ooo_plan_regions.argtypes = [c_void_p, c_int32, c_int32, c_void_p]
    lib.ooo_region_plan.restype = S
    lib.ooo_region_plan.argtypes = [c_void_p, POINTER(c_int32), POINTER(c_int32), POINTER(c_int32),
                                    POINTER(c_int32), POINTER(c_int32), POINTER(c_double), c_int32]
    lib.ooo_get_unique_id.restype = S
    lib.ooo_get_unique_id.argtypes = [c_void_p]
    lib.ooo_create_stack.restype = S
    lib.ooo_create_stack.argtypes = [POINTER(StackDesc), POINTER(c_void_p)]
    lib.ooo_forward.restype = S
    lib.ooo_forward.argtypes = [c_void_p, c_void_p, c_void_p, c_void_p]
    lib.ooo_backward.restype = S
    lib.ooo_backward.argtypes = [c_void_p, c_void_p, Schedule, c_void_p, c_void_p]
    lib.ooo_join.restype = S
    lib.ooo_join.argtypes = [c_void_p, c_void_p]
    lib.ooo_allreduce_buckets.restype = S
    lib.ooo_allreduce_buckets.argtypes = [c_void_p, c_void_p]
    lib.ooo_graph_create.restype = S
    lib.ooo_graph_create.argtypes = [c_void_p, c_void_p, c_void_p, c_void_p, Schedule, c_void_p,
                                     POINTER(c_void_p)]
    lib.ooo_graph_launch.restype = S
    lib.ooo_graph_launch.argtypes = [c_void_p, c_void_p]
    lib.ooo_graph_destroy.restype = S
    lib.ooo_graph_destroy.argtypes = [c_void_p]
    lib.ooo_destroy.restype = S
    lib.ooo_destroy.argtypes = [c_void_p]
    lib.ooo_tensor.restype = S
    lib.ooo_tensor.argtypes = [c_void_p, c_int32, c_int32, POINTER(c_void_p), POINTER(c_int64)]
    lib.ooo_set_timing.restype = S
    lib.ooo_set_timing.argtypes = [c_void_p, c_int32]
    lib.ooo_graph_upload.restype = S
    lib.ooo_graph_upload.argtypes = [c_void_p, c_void_p, c_void_p, c_void_p]
    lib.ooo_graph_launch_host.restype = S
    lib.ooo_graph_launch_host.argtypes = [c_void_p, c_void_p, c_void_p, c_void_p]
    lib.ooo_input_grad_wait.restype = S
    lib.ooo_input_grad_wait.argtypes = [c_void_p, c_void_p]
    lib.ooo_pipeline_query_sizes.restype = S
    lib.ooo_pipeline_query_sizes.argtypes = [POINTER(PipelineDesc), POINTER(c_size_t), POINTER(c_size_t)]
    lib.ooo_pipeline_grads_offset.restype = S
    lib.ooo_pipeline_grads_offset.argtypes = [POINTER(PipelineDesc), c_int32, POINTER(c_int64)]
    lib.ooo_pipeline_create.restype = S
    lib.ooo_pipeline_create.argtypes = [POINTER(PipelineDesc), POINTER(c_void_p)]
    lib.ooo_pipeline_graph_create.restype = S
    lib.ooo_pipeline_graph_create.argtypes = [c_void_p, c_void_p, c_void_p, c_void_p, c_int32, POINTER(c_void_p)]
    lib.ooo_pipeline_stage_of.restype = c_int32
    lib.ooo_pipeline_stage_of.argtypes = [c_void_p, c_int32]
    lib.ooo_pipeline_destroy.restype = S
    lib.ooo_pipeline_destroy.argtypes = [c_void_p]
    lib.ooo_comm_issue_order.restype = S
    lib.ooo_comm_issue_order.argtypes = [c_void_p, POINTER(c_int32), POINTER(c_int32), c_int32, POINTER(c_int32)]
    lib.ooo_comm_schedule.restype = S
    lib.ooo_comm_schedule.argtypes = [c_int32, POINTER(c_double), POINTER(c_int32), POINTER(c_double),
                                      POINTER(c_int32), POINTER(c_int32), c_int32, POINTER(c_int32),
                                      POINTER(c_int32), POINTER(c_double)]
    lib.ooo_graph_set_timing_slots.restype = S
    lib.ooo_graph_set_timing_slots.argtypes = [c_void_p, c_int32]
    lib.ooo_graph_timing_read.restype = S
    lib.ooo_graph_timing_read.argtypes = [c_void_p, POINTER(LaunchRecord), c_int32, POINTER(c_int32),
                                          POINTER(c_int32)]
    lib.ooo_timing_read.restype = S
    lib.ooo_timing_read.argtypes = [c_void_p, POINTER(LaunchRecord), c_int32, POINTER(c_int32)]
    _lib = lib
    return lib


def check(status: int) -> None:
    if status != OOO_OK:
        msg = load().ooo_last_error()
        raise OooError(status, msg.decode() if msg else "")


def schedule(kind: str | int, k: int = 0) -> Schedule:
    if isinstance(kind, str):
        kind = {"in_order": SCHED_IN_ORDER, "first_k": SCHED_FIRST_K, "ooo_first_k": SCHED_FIRST_K,
                "regions": SCHED_REGIONS}[kind]
    return Schedule(int(kind), int(k))
