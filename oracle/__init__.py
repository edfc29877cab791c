"""ORACLE -- test infrastructure only.

Plain, slow, obviously-correct CPU implementations of what the Paella hot path
computes, written from the paper and SURVEY.md §8(c):

* ``oracle.infer``  -- C1: float64 numpy inference of every model (plain definition).
* ``oracle.sim``    -- C2: discrete-event simulator + scheduling-policy reference
                       (SRPT on remaining time, deficit fairness, FIFO), synthetic and
                       replay modes.
* ``oracle.ringcheck`` -- C3: notification-record decoding, the reference ring
                       consumer (lap tags, torn reads), globaltimer -> host time,
                       record-time windows; exactly-once coverage (from ``sim``).
* ``oracle.eventlog`` -- reader of the dispatcher's event / routing logs.
* ``oracle.bf16``   -- RNE float32 -> bfloat16, the ingest rounding.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import anything in this package.  It shares no code
with ``paper_conf_sosp_ngd023_b200/`` (the CUDA path); both read their inputs from
the neutral ``workload`` package.
"""
