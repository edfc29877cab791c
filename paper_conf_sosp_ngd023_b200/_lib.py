"""Thin ctypes binding of ``include/paella.h`` (argument marshalling only).

Every step of the hot path -- admission, scheduling, launches, kernels, completion
-- runs in ``libpaella.so``; this module only converts Python values to the C
structs and back.  It fails loudly when the library is missing: there is no
Python or CPU fallback of the GPU path.
"""
from __future__ import annotations

import ctypes as C
import errno
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# PAELLA_LIB: another build of the same library (the ThreadSanitizer build, build.py --tsan)
LIB_PATH = os.environ.get("PAELLA_LIB") or os.path.join(HERE, "libpaella.so")

ABI_VERSION = 2
NOTIFY_COUNTERS, NOTIFY_RING = 0, 1
POLICY_SRPT_DEFICIT, POLICY_FIFO, POLICY_SJF, POLICY_RR = 0, 1, 2, 3
ROUTE_LEAST_WORK, ROUTE_ROUND_ROBIN, ROUTE_POWER_OF_TWO = 0, 1, 2
DEVICE_CUDA, DEVICE_FAKE = 0, 1
DTYPE_BF16, DTYPE_FP32 = 0, 1
NONBLOCK = 1
FAULT_NONE, FAULT_DROP, FAULT_DUP, FAULT_TORN, FAULT_HANG, FAULT_CORRUPT = 0, 1, 2, 3, 4, 5
HYBRID = 2
OP = {"input": 0, "conv": 1, "maxpool": 2, "avgpool": 3, "gap": 4, "fc": 5, "concat": 6, "spin": 7}
ACT = {"none": 0, "relu": 1, "relu6": 2}
NODE_PROLOGUE, NODE_CEIL = 1, 2
INT64_MAX = (1 << 63) - 1

#: every symbol include/paella.h declares
SYMBOLS = ["paella_init", "paella_register_model", "paella_submit", "paella_submit_at",
           "paella_poll_completion", "paella_shutdown", "paella_client_region", "paella_model_info",
           "paella_kernel_info", "paella_kernel_name", "paella_stats", "paella_flush_log",
           "paella_run_isolated", "paella_debug_node", "paella_time_kernels", "paella_bench_empty",
           "paella_bench_roundtrip", "paella_loadgen", "paella_bench_wait", "paella_route_pair",
           "paella_clock_info", "paella_clock_sync", "paella_channel_path", "paella_client_attach",
           "paella_client_region_of", "paella_client_model_io", "paella_client_submit", "paella_client_poll",
           "paella_client_detach", "paella_bench_xdev", "paella_check_counters"]


class Config(C.Structure):
    _fields_ = [("abi_version", C.c_uint32), ("device", C.c_uint32), ("num_gpus", C.c_uint32),
                ("first_gpu", C.c_uint32), ("num_clients", C.c_uint32), ("policy", C.c_uint32),
                ("fairness_threshold", C.c_int64), ("slack_blocks", C.c_uint32), ("group_size", C.c_uint32),
                ("ring_capacity", C.c_uint32), ("stream_pool", C.c_uint32), ("route", C.c_uint32),
                ("submit_slots", C.c_uint32), ("max_jobs_per_model", C.c_uint32), ("instrument", C.c_uint32),
                ("naive", C.c_uint32), ("client_region_bytes", C.c_size_t),
                ("dispatcher_cpus", C.POINTER(C.c_int32)), ("event_log_path", C.c_char_p),
                ("fake_sms", C.c_uint32), ("fake_time_scale_ns", C.c_uint32), ("event_time_kind", C.c_uint32),
                ("lookahead", C.c_uint32), ("launch_threads", C.c_uint32),
                ("no_proxy", C.c_uint32), ("no_pdl", C.c_uint32),
                ("notify_mode", C.c_uint32), ("prio_classes", C.c_uint32), ("online_tbar", C.c_uint32),
                ("decide_delay_ns", C.c_uint32), ("naive_pdl", C.c_uint32), ("watchdog_ms", C.c_uint32),
                ("fake_fault", C.c_uint32), ("fake_fault_arg", C.c_uint32), ("branches", C.c_uint32),
                ("route_log_path", C.c_char_p),
                ("max_active_jobs", C.c_uint32), ("lookahead_unplaced", C.c_uint32),
                ("cap_arrival_order", C.c_uint32)]


class Node(C.Structure):
    _fields_ = [("op", C.c_uint32), ("n_inputs", C.c_uint32), ("inputs", C.POINTER(C.c_int32)),
                ("residual", C.c_int32), ("c", C.c_uint32), ("h", C.c_uint32), ("w", C.c_uint32),
                ("cout", C.c_uint32), ("kh", C.c_uint32), ("kw", C.c_uint32), ("sh", C.c_uint32),
                ("sw", C.c_uint32), ("ph", C.c_uint32), ("pw", C.c_uint32), ("groups", C.c_uint32),
                ("act", C.c_uint32), ("flags", C.c_uint32), ("weight", C.POINTER(C.c_float)),
                ("bias", C.POINTER(C.c_float)), ("pro_scale", C.POINTER(C.c_float)),
                ("pro_shift", C.POINTER(C.c_float))]


class ModelDesc(C.Structure):
    _fields_ = [("name", C.c_char_p), ("dtype", C.c_uint32), ("n_nodes", C.c_uint32),
                ("nodes", C.POINTER(Node)), ("profile_runs", C.c_uint32)]


class ModelInfo(C.Structure):
    _fields_ = [("n_kernels", C.c_uint32), ("input_bytes", C.c_size_t), ("output_bytes", C.c_size_t),
                ("weight_bytes", C.c_uint64), ("total_tbar_ns", C.c_int64)]


class KernelInfo(C.Structure):
    _fields_ = [("grid", C.c_uint32), ("block", C.c_uint32), ("smem", C.c_uint32), ("regs", C.c_uint32),
                ("tmem_cols", C.c_uint32), ("kind", C.c_uint32), ("tbar_ns", C.c_int64),
                ("flops", C.c_uint64), ("bytes", C.c_uint64), ("vs", C.c_uint32), ("n_deps", C.c_uint32),
                ("deps", C.c_uint32 * 8)]


class Req(C.Structure):
    _fields_ = [("t_ns", C.c_int64), ("client", C.c_uint32), ("model", C.c_uint32),
                ("input_idx", C.c_uint32), ("pad", C.c_uint32)]


class Stats(C.Structure):
    _fields_ = [("admitted", C.c_uint64), ("completed", C.c_uint64), ("launches", C.c_uint64),
                ("records", C.c_uint64), ("torn_retries", C.c_uint64), ("decide_calls", C.c_uint64),
                ("loop_iters", C.c_uint64), ("outstanding_work_ns", C.c_int64), ("ev_launches", C.c_uint64),
                ("ev_ns", C.c_uint64), ("ev_bytes", C.c_uint64), ("ev_flops", C.c_uint64),
                ("stop_reason", C.c_uint64 * 5), ("sum_ready", C.c_uint64), ("sum_live_jobs", C.c_uint64),
                ("sum_Q", C.c_uint64), ("rel_events", C.c_uint64), ("xstream_waits", C.c_uint64),
                ("busy_ns", C.c_uint64)]


_lib = None


def load():
    """Load libpaella.so (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} missing: run `python -m paper_conf_sosp_ngd023_b200.build` "
                           "(there is no CPU fallback of the CUDA path)")
    lib = C.CDLL(LIB_PATH)
    P = C.c_void_p
    lib.paella_init.argtypes = [C.POINTER(Config), C.POINTER(P)]
    lib.paella_register_model.argtypes = [P, C.POINTER(ModelDesc), C.POINTER(C.c_uint32)]
    lib.paella_submit.argtypes = [P, C.c_uint32, C.c_uint32, P, C.c_size_t, C.c_uint32]
    lib.paella_submit.restype = C.c_int64
    lib.paella_submit_at.argtypes = [P, C.c_uint32, C.c_uint32, P, C.c_size_t, C.c_uint32, C.c_int64]
    lib.paella_submit_at.restype = C.c_int64
    lib.paella_poll_completion.argtypes = [P, C.c_uint32, C.c_uint32, C.POINTER(C.c_int32)]
    lib.paella_poll_completion.restype = C.c_int64
    lib.paella_shutdown.argtypes = [P]
    lib.paella_route_pair.argtypes = [C.c_uint64, C.c_uint32, C.POINTER(C.c_uint32), C.POINTER(C.c_uint32)]
    lib.paella_client_region.argtypes = [P, C.c_uint32, C.POINTER(P), C.POINTER(C.c_size_t)]
    lib.paella_model_info.argtypes = [P, C.c_uint32, C.POINTER(ModelInfo)]
    lib.paella_kernel_info.argtypes = [P, C.c_uint32, C.c_uint32, C.POINTER(KernelInfo)]
    lib.paella_kernel_name.argtypes = [C.c_uint32]
    lib.paella_kernel_name.restype = C.c_char_p
    lib.paella_stats.argtypes = [P, C.c_uint32, C.POINTER(Stats)]
    lib.paella_clock_info.argtypes = [P, C.c_uint32, C.POINTER(C.c_int64), C.POINTER(C.c_int64),
                                      C.POINTER(C.c_int64)]
    lib.paella_clock_sync.argtypes = [P, C.c_uint32]
    lib.paella_check_counters.argtypes = [P, C.c_uint32, C.POINTER(C.c_uint32)]
    lib.paella_channel_path.argtypes = [P, C.c_char_p, C.c_size_t]
    lib.paella_bench_xdev.argtypes = [P, C.c_uint32, C.POINTER(C.c_uint32), C.c_uint32, C.POINTER(C.c_uint32),
                                      C.c_uint32, C.c_uint32, C.POINTER(C.c_double)]
    lib.paella_client_attach.argtypes = [C.c_char_p, C.c_uint32, C.POINTER(P)]
    lib.paella_client_region_of.argtypes = [P, C.POINTER(P), C.POINTER(C.c_size_t)]
    lib.paella_client_model_io.argtypes = [P, C.c_uint32, C.POINTER(C.c_size_t), C.POINTER(C.c_size_t)]
    lib.paella_client_submit.argtypes = [P, C.c_uint32, P, C.c_size_t, C.c_uint32]
    lib.paella_client_submit.restype = C.c_int64
    lib.paella_client_poll.argtypes = [P, C.c_uint32, C.POINTER(C.c_int32)]
    lib.paella_client_poll.restype = C.c_int64
    lib.paella_client_detach.argtypes = [P]
    lib.paella_flush_log.argtypes = [P]
    lib.paella_run_isolated.argtypes = [P, C.c_uint32, C.c_uint32, P, P, C.POINTER(C.c_int64)]
    lib.paella_debug_node.argtypes = [P, C.c_uint32, C.c_uint32, C.c_uint32, C.POINTER(C.c_float)]
    lib.paella_time_kernels.argtypes = [P, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, C.POINTER(C.c_int64)]
    lib.paella_bench_empty.argtypes = [P, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32,
                                       C.POINTER(C.c_double)]
    lib.paella_bench_roundtrip.argtypes = [P, C.c_uint32, C.c_uint32, C.POINTER(C.c_int64), C.POINTER(C.c_int64)]
    lib.paella_loadgen.argtypes = [P, C.POINTER(Req), C.c_uint32, C.c_size_t, C.c_uint32, P, C.c_int64,
                                   C.POINTER(C.c_int64), C.POINTER(C.c_int64)]
    lib.paella_loadgen.restype = C.c_int64
    lib.paella_bench_wait.argtypes = [P, C.c_uint32, C.c_uint32, C.c_uint32, C.c_int64, C.c_uint32, C.c_size_t,
                                      C.c_uint32, C.POINTER(C.c_int64), C.POINTER(C.c_double)]
    lib.paella_bench_wait.restype = C.c_int
    _lib = lib
    return lib


def _check(rc, what):
    if rc < 0:
        raise OSError(-rc, f"{what}: {os.strerror(-rc)}")
    return rc


def _fptr(a):
    return a.ctypes.data_as(C.POINTER(C.c_float)) if a is not None else None


def route_pair(req_id, num_gpus):
    """``paella_route_pair``: the two candidate GPUs of ROUTE_POWER_OF_TWO."""
    g0, g1 = C.c_uint32(), C.c_uint32()
    _check(load().paella_route_pair(req_id, num_gpus, C.byref(g0), C.byref(g1)), "paella_route_pair")
    return g0.value, g1.value


class Engine:
    """One Paella instance (``paella_init`` ... ``paella_shutdown``)."""

    def __init__(self, num_clients=1, num_gpus=1, first_gpu=0, device=DEVICE_CUDA,
                 policy=POLICY_SRPT_DEFICIT, theta=100, slack=0, group=16, ring_capacity=65536,
                 streams=32, route=ROUTE_LEAST_WORK, submit_slots=1024, max_jobs_per_model=128,
                 instrument=True, naive=False, region_bytes=64 << 20, dispatcher_cpus=None,
                 event_log=None, fake_sms=0, fake_time_scale_ns=0, event_time_kind=None, lookahead=0,
                 launch_threads=0, proxy=True, pdl=True, prio_classes=1,
                 notify="counters", decide_delay_ns=0, online_tbar=False, naive_pdl=False, watchdog_ms=0,
                 fake_fault=0, fake_fault_arg=0, route_log=None, max_active=0, branches=False,
                 lookahead_unplaced=False, cap_fifo=False):
        self.lib = load()
        cfg = Config()
        cfg.abi_version = ABI_VERSION
        cfg.device = device
        cfg.num_gpus = num_gpus
        cfg.first_gpu = first_gpu
        cfg.num_clients = num_clients
        cfg.policy = policy
        cfg.fairness_threshold = INT64_MAX if theta is None else theta
        cfg.slack_blocks = slack
        cfg.group_size = group
        cfg.ring_capacity = ring_capacity
        cfg.stream_pool = streams
        cfg.route = route
        cfg.submit_slots = submit_slots
        cfg.max_jobs_per_model = max_jobs_per_model
        cfg.instrument = 1 if instrument else 0
        cfg.naive = 1 if naive else 0
        cfg.client_region_bytes = region_bytes
        self._cpus = None
        if dispatcher_cpus is not None:
            self._cpus = (C.c_int32 * len(dispatcher_cpus))(*dispatcher_cpus)
            cfg.dispatcher_cpus = self._cpus
        self._log = event_log.encode() if event_log else None
        cfg.event_log_path = self._log
        cfg.fake_sms = fake_sms
        cfg.fake_time_scale_ns = fake_time_scale_ns
        cfg.event_time_kind = 0 if event_time_kind is None else event_time_kind + 1
        cfg.lookahead = lookahead
        cfg.launch_threads = launch_threads
        cfg.no_proxy = 0 if proxy else 1
        cfg.no_pdl = 0 if pdl else 1
        cfg.prio_classes = prio_classes
        cfg.decide_delay_ns = decide_delay_ns
        cfg.online_tbar = 1 if online_tbar else 0
        cfg.naive_pdl = 1 if naive_pdl else 0
        cfg.watchdog_ms = watchdog_ms
        cfg.fake_fault = fake_fault
        cfg.fake_fault_arg = fake_fault_arg
        self._rlog = route_log.encode() if route_log else None
        cfg.route_log_path = self._rlog
        cfg.max_active_jobs = max_active
        cfg.lookahead_unplaced = 1 if lookahead_unplaced else 0
        cfg.cap_arrival_order = 1 if cap_fifo else 0
        cfg.branches = 1 if branches else 0
        # notification path: "counters" (default), "ring" (device ring + forwarding warp),
        # "direct" (the paper's direct ring writes; same as proxy=False)
        if notify not in ("counters", "ring", "direct"):
            raise ValueError(notify)
        cfg.notify_mode = NOTIFY_RING if notify == "ring" else NOTIFY_COUNTERS
        if notify == "direct":
            cfg.no_proxy = 1
        self.cfg = cfg
        h = C.c_void_p()
        _check(self.lib.paella_init(C.byref(cfg), C.byref(h)), "paella_init")
        self.h = h
        self.num_clients = num_clients
        self._keep = []
        self._regions = {}

    # -- models --------------------------------------------------------------
    def register_model(self, graph, params, dtype=DTYPE_BF16, name=None):
        """Marshal a workload.archs.Graph + {name: array} into paella_node_t[]."""
        keep = []
        nodes = (Node * len(graph.nodes))()
        for i, n in enumerate(graph.nodes):
            nd = nodes[i]
            nd.op = OP[n["op"]]
            ins = np.asarray(n["inputs"], dtype=np.int32)
            keep.append(ins)
            nd.n_inputs = len(ins)
            nd.inputs = ins.ctypes.data_as(C.POINTER(C.c_int32)) if len(ins) else None
            nd.residual = -1 if n.get("residual") is None else n["residual"]
            nd.c, nd.h, nd.w = n["out"]
            nd.act = ACT[n.get("act", "none")]
            flags = 0
            if n.get("prologue"):
                flags |= NODE_PROLOGUE
            if n.get("ceil"):
                flags |= NODE_CEIL
            nd.flags = flags
            if n["op"] == "conv":
                nd.cout, nd.kh, nd.kw = n["cout"], n["kh"], n["kw"]
                nd.sh, nd.sw, nd.ph, nd.pw, nd.groups = n["sh"], n["sw"], n["ph"], n["pw"], n["groups"]
            elif n["op"] in ("maxpool", "avgpool"):
                nd.kh = nd.kw = n["k"]
                nd.sh = nd.sw = n["s"]
                nd.ph = nd.pw = n["p"]
                nd.groups = 1
            elif n["op"] == "fc":
                nd.cout = n["cout"]
            elif n["op"] == "spin":
                nd.kh = n["us"]
            if n["op"] in ("conv", "fc"):
                w = np.ascontiguousarray(params[n["name"] + ".weight"], dtype=np.float32)
                b = np.ascontiguousarray(params[n["name"] + ".bias"], dtype=np.float32)
                keep += [w, b]
                nd.weight, nd.bias = _fptr(w), _fptr(b)
            if n.get("prologue"):
                s = np.ascontiguousarray(params[n["name"] + ".pro_scale"], dtype=np.float32)
                z = np.ascontiguousarray(params[n["name"] + ".pro_shift"], dtype=np.float32)
                keep += [s, z]
                nd.pro_scale, nd.pro_shift = _fptr(s), _fptr(z)
        desc = ModelDesc()
        nm = (name or graph.name).encode()
        desc.name = nm
        desc.dtype = dtype
        desc.n_nodes = len(graph.nodes)
        desc.nodes = nodes
        mid = C.c_uint32()
        _check(self.lib.paella_register_model(self.h, C.byref(desc), C.byref(mid)), "paella_register_model")
        return mid.value

    def model_info(self, mid):
        info = ModelInfo()
        _check(self.lib.paella_model_info(self.h, mid, C.byref(info)), "paella_model_info")
        return {f: getattr(info, f) for f, _ in ModelInfo._fields_}

    def kernel_info(self, mid, k):
        info = KernelInfo()
        _check(self.lib.paella_kernel_info(self.h, mid, k, C.byref(info)), "paella_kernel_info")
        d = {f: getattr(info, f) for f, _ in KernelInfo._fields_}
        d["deps"] = list(info.deps)[:min(8, info.n_deps)]
        d["name"] = self.lib.paella_kernel_name(info.kind).decode()
        return d

    def kernels(self, mid):
        return [self.kernel_info(mid, k) for k in range(self.model_info(mid)["n_kernels"])]

    # -- client channel --------------------------------------------------------
    def region(self, client):
        """The client's shared io region as a uint8 numpy array (zero-copy)."""
        if client not in self._regions:
            base, size = C.c_void_p(), C.c_size_t()
            _check(self.lib.paella_client_region(self.h, client, C.byref(base), C.byref(size)),
                   "paella_client_region")
            buf = (C.c_uint8 * size.value).from_address(base.value)
            self._regions[client] = (base.value, np.frombuffer(buf, dtype=np.uint8))
        return self._regions[client]

    def submit(self, client, model, io_off, length, flags=0, t_sched_ns=None):
        base, _ = self.region(client)
        if t_sched_ns is None:
            return self.lib.paella_submit(self.h, client, model, base + io_off, length, flags)
        return self.lib.paella_submit_at(self.h, client, model, base + io_off, length, flags, t_sched_ns)

    def poll(self, client, flags=NONBLOCK):
        st = C.c_int32()
        rid = self.lib.paella_poll_completion(self.h, client, flags, C.byref(st))
        return rid, st.value

    # -- isolated runs / introspection ----------------------------------------------
    def run_isolated(self, model, image, gpu=0, timing=False):
        info = self.model_info(model)
        x = np.ascontiguousarray(image, dtype=np.float32)
        assert x.nbytes == info["input_bytes"], (x.nbytes, info["input_bytes"])
        out = np.zeros(info["output_bytes"] // 4, dtype=np.float32)
        kt = np.zeros(info["n_kernels"], dtype=np.int64) if timing else None
        _check(self.lib.paella_run_isolated(self.h, gpu, model, x.ctypes.data, out.ctypes.data,
                                            kt.ctypes.data_as(C.POINTER(C.c_int64)) if timing else None),
               "paella_run_isolated")
        return (out, kt) if timing else out

    def debug_node(self, model, node, shape, gpu=0):
        out = np.zeros(int(np.prod(shape)), dtype=np.float32)
        _check(self.lib.paella_debug_node(self.h, gpu, model, node, _fptr(out)), "paella_debug_node")
        return out.reshape(shape)

    def time_kernels(self, model, instrumented=True, reps=50, gpu=0, l2_cold=False):
        n = self.model_info(model)["n_kernels"]
        kt = np.zeros(n, dtype=np.int64)
        flags = (1 if instrumented else 0) | (2 if l2_cold else 0)
        _check(self.lib.paella_time_kernels(self.h, gpu, model, flags, reps,
                                            kt.ctypes.data_as(C.POINTER(C.c_int64))), "paella_time_kernels")
        return kt

    def bench_empty(self, grid, block=128, instrumented=True, group=16, iters=2000, gpu=0):
        v = C.c_double()
        _check(self.lib.paella_bench_empty(self.h, gpu, grid, block, 1 if instrumented else 0, group, iters,
                                           C.byref(v)), "paella_bench_empty")
        return v.value

    def bench_roundtrip(self, n=1000, gpu=0):
        a = np.zeros(n, dtype=np.int64)
        b = np.zeros(n, dtype=np.int64)
        _check(self.lib.paella_bench_roundtrip(self.h, gpu, n, a.ctypes.data_as(C.POINTER(C.c_int64)),
                                               b.ctypes.data_as(C.POINTER(C.c_int64))), "paella_bench_roundtrip")
        return a, b

    def bench_xdev(self, models, seq, streams=32, gpu=0):
        """X_dev: device-only saturation req/s of the mix (paella_bench_xdev)."""
        ms = (C.c_uint32 * len(models))(*models)
        sq = (C.c_uint32 * len(seq))(*[int(x) for x in seq])
        v = C.c_double()
        _check(self.lib.paella_bench_xdev(self.h, gpu, ms, len(models), sq, len(seq), streams, C.byref(v)),
               "paella_bench_xdev")
        return v.value

    def bench_wait(self, client, model, n, gap_ns, poll_flags, stride, slots):
        """NEXT-3 measurement: (jct_ns array, waiter CPU fraction); see paella_bench_wait."""
        j = np.zeros(n, dtype=np.int64)
        f = C.c_double()
        _check(self.lib.paella_bench_wait(self.h, client, model, n, int(gap_ns), poll_flags, stride, slots,
                                          j.ctypes.data_as(C.POINTER(C.c_int64)), C.byref(f)), "paella_bench_wait")
        return j, f.value

    def loadgen(self, t_ns, clients, models, inputs, stride, slots, copy_inputs=None, t0_ns=0):
        """Open-loop replay of a trace from the calling thread (GIL released).
        copy_inputs: None (inputs pre-staged in the slots) or {model: [np arrays]}.
        Returns (jct_ns array, elapsed_ns)."""
        n = len(t_ns)
        reqs = (Req * n)()
        for i in range(n):
            reqs[i].t_ns = int(t_ns[i])
            reqs[i].client = int(clients[i])
            reqs[i].model = int(models[i])
            reqs[i].input_idx = int(inputs[i])
        jct = np.zeros(n, dtype=np.int64)
        el = C.c_int64()
        cp = None
        if copy_inputs is not None:
            nm = max(copy_inputs) + 1
            rows = (C.c_void_p * nm)()
            self._cp_keep = []
            for m, arrs in copy_inputs.items():
                ptrs = (C.c_void_p * len(arrs))(*[a.ctypes.data for a in arrs])
                self._cp_keep.append((ptrs, arrs))
                rows[m] = C.cast(ptrs, C.c_void_p)
            cp = rows
            self._cp_keep.append(rows)
        rc = self.lib.paella_loadgen(self.h, reqs, n, stride, slots, C.cast(cp, C.c_void_p) if cp else None,
                                     t0_ns, jct.ctypes.data_as(C.POINTER(C.c_int64)), C.byref(el))
        _check(rc, "paella_loadgen")
        return jct, el.value

    def stats(self, gpu=0):
        st = Stats()
        _check(self.lib.paella_stats(self.h, gpu, C.byref(st)), "paella_stats")
        d = {f: getattr(st, f) for f, _ in Stats._fields_}
        d["stop_reason"] = list(st.stop_reason)
        return d

    def clock_info(self, gpu=0):
        """(offset_ns, rtt_ns, resolution_ns) of the globaltimer -> host calibration."""
        o, r, q = C.c_int64(), C.c_int64(), C.c_int64()
        _check(self.lib.paella_clock_info(self.h, gpu, C.byref(o), C.byref(r), C.byref(q)), "paella_clock_info")
        return o.value, r.value, q.value

    def channel_path(self):
        """Path another process passes to Client() to attach to this instance."""
        buf = C.create_string_buffer(256)
        _check(self.lib.paella_channel_path(self.h, buf, 256), "paella_channel_path")
        return buf.value.decode()

    def check_counters(self, gpu=0):
        """(mismatching slots, slots used): paella_check_counters."""
        n = C.c_uint32()
        bad = _check(self.lib.paella_check_counters(self.h, gpu, C.byref(n)), "paella_check_counters")
        return bad, n.value

    def clock_sync(self, gpu=0):
        _check(self.lib.paella_clock_sync(self.h, gpu), "paella_clock_sync")

    def flush_log(self):
        self.lib.paella_flush_log(self.h)

    def shutdown(self):
        if self.h:
            rc = self.lib.paella_shutdown(self.h)
            self.h = None
            self._regions.clear()
            return rc
        return 0

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.shutdown()


class Client:
    """A client in ANOTHER process (``paella_client_attach``): the same zero-copy
    predict / readResult channel as Engine.submit / Engine.poll."""

    def __init__(self, path, client_id):
        self.lib = load()
        h = C.c_void_p()
        _check(self.lib.paella_client_attach(path.encode(), client_id, C.byref(h)), "paella_client_attach")
        self.h = h
        base, size = C.c_void_p(), C.c_size_t()
        _check(self.lib.paella_client_region_of(self.h, C.byref(base), C.byref(size)), "paella_client_region_of")
        self.base = base.value
        self.region = np.frombuffer((C.c_uint8 * size.value).from_address(base.value), dtype=np.uint8)

    def model_io(self, model):
        i, o = C.c_size_t(), C.c_size_t()
        _check(self.lib.paella_client_model_io(self.h, model, C.byref(i), C.byref(o)), "paella_client_model_io")
        return i.value, o.value

    def submit(self, model, io_off, length, flags=0):
        return self.lib.paella_client_submit(self.h, model, self.base + io_off, length, flags)

    def poll(self, flags=NONBLOCK):
        st = C.c_int32()
        rid = self.lib.paella_client_poll(self.h, flags, C.byref(st))
        return rid, st.value

    def close(self):
        if self.h:
            self.region = None
            self.lib.paella_client_detach(self.h)
            self.h = None


EAGAIN = errno.EAGAIN
