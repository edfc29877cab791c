"""ORACLE (test infrastructure) -- C3: notification-record decoding and ring checks.

Paper: the notification queue entry {type, smId, kernId} (P1126-1133), the INVALID
reset of consumed slots (P1107-1113), group records of up to 16 blocks (P1138-1142);
readings C2-Q3..Q5 fix the 16-byte record:

    w0 = type:8 | count:8 | smid:8 | tag:8 | uid:32            (bit 0 = LSB)
    w1 = gtimer_ns:40 | group:16 | tag:8            tag = 0x80 | (lap & 0x7f)

where lap = ring index >> log2(capacity) and type 0 = INVALID.  A slot is consumable
when its type is not INVALID and BOTH halves carry the tag of the consumer's current
lap; if w0 has it and w1 does not, the record is torn (its second half has not landed)
and must be re-read later, never consumed.

Written from that specification only; it shares no code with the CUDA path
(paper_conf_sosp_ngd023_b200/csrc/common.h), which the tests compare against it on
real and fake-device rings.  Exactly-once coverage is ``oracle.sim.check_exactly_once``
(re-exported here).  Only tests/ may import this module.
"""
from __future__ import annotations

from .sim import check_exactly_once  # noqa: F401  (C3 coverage check lives with S5)

INVALID, PLACEMENT, COMPLETION = 0, 1, 2
GTIMER_BITS = 40


def tag(lap):
    return 0x80 | (lap & 0x7F)


def decode(w0, w1):
    """Fields of one record (dict)."""
    return dict(type=w0 & 0xFF, count=(w0 >> 8) & 0xFF, smid=(w0 >> 16) & 0xFF, tag0=(w0 >> 24) & 0xFF,
                uid=(w0 >> 32) & 0xFFFFFFFF, gtimer=w1 & ((1 << GTIMER_BITS) - 1), group=(w1 >> 40) & 0xFFFF,
                tag1=(w1 >> 56) & 0xFF)


def consume(words, head, log2cap):
    """Reference consumer of a ring snapshot.

    words: sequence of (w0, w1) per slot (len = capacity); head: the consumer's ring
    index.  Returns (records consumed in order, new head, torn) where torn is True if
    the scan stopped at a torn slot (valid first half of the current lap, second half
    not yet)."""
    cap = 1 << log2cap
    out = []
    while True:
        w0, w1 = words[head & (cap - 1)]
        want = tag(head >> log2cap)
        if (w0 & 0xFF) == INVALID or ((w0 >> 24) & 0xFF) != want:
            return out, head, False
        if ((w1 >> 56) & 0xFF) != want:
            return out, head, True
        out.append(decode(w0, w1))
        head += 1


def device_to_host_ns(gtimer40, offset_ns, ref_host_ns):
    """Host CLOCK_MONOTONIC time of a record's 40-bit %globaltimer field.

    The device time is gtimer40 + k * 2^40 for the k that puts it closest to the
    device time of a reference host instant (ref_host_ns + offset_ns); then
    host = device - offset (offset = globaltimer - host, paella_clock_info)."""
    span = 1 << GTIMER_BITS
    ref_dev = ref_host_ns + offset_ns
    k = (ref_dev - gtimer40 + span // 2) // span
    return gtimer40 + k * span - offset_ns


def offset_at(clocks, host_ns):
    """globaltimer - host offset at host time host_ns: linear interpolation between the
    calibrations (dicts with 'at' = host time of the sample, 'offset'), extrapolated with
    the nearest segment; one calibration = a constant offset (the clocks drift by ppm)."""
    cs = sorted(clocks, key=lambda c: c["at"])
    if len(cs) == 1:
        return cs[0]["offset"]
    i = 0
    while i + 2 < len(cs) and host_ns > cs[i + 1]["at"]:
        i += 1
    a, b = cs[i], cs[i + 1]
    return a["offset"] + (b["offset"] - a["offset"]) * (host_ns - a["at"]) / max(1, b["at"] - a["at"])


def check_record_times(records, windows, clocks, tol_ns):
    """Every record of a launch, converted to host time, must fall inside the life of
    the job that issued it: [scheduled arrival - tol, completion seen by the dispatcher
    + tol].

    records: (gtimer40, type, uid, count, group[, smid]) as eventlog extras["records"];
    windows: uid -> (t_sched, t_complete) in host CLOCK_MONOTONIC ns; clocks: the
    calibrations (offset_at), or one offset.  Returns the violations (uid, ns after
    arrival, ns before completion)."""
    if not isinstance(clocks, (list, tuple)):
        clocks = [{"at": 0, "offset": clocks}]
    bad = []
    for r in records:
        t40, uid = r[0], r[2]
        t_arr, t_done = windows[uid]
        t = device_to_host_ns(t40, round(offset_at(clocks, t_done)), t_done)
        if not t_arr - tol_ns <= t <= t_done + tol_ns:
            bad.append((uid, t - t_arr, t_done - t))
    return bad
