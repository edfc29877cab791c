"""Pins for oracle C3 (oracle/ringcheck.py): the record layout decoded from hand-encoded
bit patterns, the reference consumer on hand-built rings (valid / torn / stale-lap /
INVALID slots), and the globaltimer -> host conversion across the 40-bit wrap."""
from oracle import ringcheck as rc


def enc(typ, count, smid, lap, uid, gt, group):
    """Hand encoding, written from the layout table in the module docstring."""
    t = 0x80 | (lap & 0x7F)
    w0 = typ | count << 8 | smid << 16 | t << 24 | uid << 32
    w1 = gt | group << 40 | t << 56
    return w0, w1


def test_decode_hand_encoded_literal():
    # type 2, count 16, SM 147, lap 3 (tag 0x83), uid 0xDEADBEEF, gtimer 0x123456789A, group 0x0102
    w0, w1 = 0xDEADBEEF83931002, 0x830102123456789A
    d = rc.decode(w0, w1)
    assert d == dict(type=2, count=16, smid=147, tag0=0x83, uid=0xDEADBEEF, gtimer=0x123456789A,
                     group=0x0102, tag1=0x83)
    assert enc(2, 16, 147, 3, 0xDEADBEEF, 0x123456789A, 0x0102) == (w0, w1)


def test_consume_stops_at_torn_invalid_and_stale():
    log2cap = 2
    a = enc(1, 16, 0, 0, 7, 100, 0)
    b = enc(2, 16, 1, 0, 7, 200, 0)
    c = enc(1, 3, 2, 0, 8, 300, 0)
    torn = (c[0], 0)                                   # second half still the reset value
    ring = [a, b, torn, (0, 0)]
    out, head, is_torn = rc.consume(ring, 0, log2cap)
    assert [r["uid"] for r in out] == [7, 7] and head == 2 and is_torn
    ring[2] = c                                        # the second half lands
    out, head, is_torn = rc.consume(ring, 2, log2cap)
    assert [r["count"] for r in out] == [3] and head == 3 and not is_torn   # slot 3 INVALID
    # lap 1 starts at head 4: slot 0 still holds lap 0's record -> stale, not consumed
    out, head, is_torn = rc.consume([a, b, c, enc(2, 3, 0, 0, 8, 400, 0)], 4, log2cap)
    assert out == [] and head == 4 and not is_torn
    lap1 = enc(1, 1, 0, 1, 9, 500, 0)
    out, head, _ = rc.consume([lap1, b, c, c], 4, log2cap)
    assert [r["uid"] for r in out] == [9] and head == 5


def test_device_to_host_across_wrap():
    span = 1 << 40
    off = 5_000_000_123
    for host in (10**12, 3 * span - 17, 7 * span + 5):
        dev = host + off
        assert rc.device_to_host_ns(dev % span, off, host) == host
        assert rc.device_to_host_ns(dev % span, off, host + 10**9) == host   # reference 1 s later
        assert rc.device_to_host_ns((dev - 10**6) % span, off, host) == host - 10**6


def test_record_time_windows():
    off = 1000
    recs = [(2500 + off, 1, 5, 16, 0), (2900 + off, 2, 5, 16, 0)]
    assert rc.check_record_times(recs, {5: (2000, 3000)}, off, 0) == []
    assert rc.check_record_times(recs, {5: (2600, 3000)}, off, 0) != []       # before arrival
    assert rc.check_record_times(recs, {5: (2000, 2800)}, off, 50) != []      # after completion


def test_offset_interpolation():
    cl = [{"at": 1000, "offset": 100}, {"at": 3000, "offset": 300}]
    assert rc.offset_at(cl, 2000) == 200
    assert rc.offset_at(cl, 5000) == 500          # extrapolated on the last segment
    assert rc.offset_at(cl[:1], 9999) == 100
    off = lambda h: rc.offset_at(cl, h)   # noqa: E731
    recs = [(int(2500 + off(2500)), 1, 5, 16, 0)]
    assert rc.check_record_times(recs, {5: (2400, 2600)}, cl, 0) == []
