"""Test-side encoder/decoder of the Orion binary log.

Third, independent implementation of the format (the product library and oracle/policy.c each
have their own). Used to build synthetic traces for the oracle and to decode logs for comparison.
"""
import struct

MAGIC = b"ORIONLG1"
HDR_BYTES = 240
KIND = {"KERNEL": 0, "MEMCPY": 1, "MEMCPY_H2D": 1, "MEMCPY_D2H": 2, "MEMSET": 3}
CLS = {"U": 0, "C": 1, "M": 2}
DEC_NAMES = {1: "HP_LAUNCH", 2: "PASS", 3: "ADMIT_IDLE", 4: "ADMIT_COLOC", 5: "DEFER_SM",
             6: "DEFER_PROFILE", 7: "DEFER_DUR", 8: "RESET"}
DEC_CODES = {v: k for k, v in DEC_NAMES.items()}
T_VIS, T_DONE = 1, 2
FLAGS = {"HP_BUSY_REQUEST": 1, "HP_REF_ALL": 2, "HP_UNKNOWN_STRICT": 4,
         "THROTTLE_ONLY_HP_BUSY": 8, "FREE_SMS": 16}


def encode(num_sms, sm_thr, dur_thr, flags, prios, ops, tape=None, k_end=0):
    """prios: list of 0 (HP) / 1 (BE) per client. ops: list (per client) of tuples
    (kernel_id, kind, opflags, cls, sm_needed, dur_ns). tape: list of (k, type, client, value)."""
    n = len(prios)
    hp = prios.index(0) if 0 in prios else -1
    b = bytearray()
    b += MAGIC
    b += struct.pack("<IIII", 1, n, num_sms, sm_thr)
    b += struct.pack("<QIi", dur_thr, flags, hp)
    b += struct.pack("<16I", *(list(prios) + [0xFFFFFFFF] * (16 - n)))
    b += struct.pack("<Q", k_end)
    b += struct.pack("<16Q", *([len(o) for o in ops] + [0] * (16 - n)))
    assert len(b) == HDR_BYTES
    for cl in ops:
        for (kid, kind, opf, cls, sm, dur) in cl:
            b += struct.pack("<IHBBIIQ", kid, kind, opf, cls, sm, 0, dur)
    if tape is not None:
        b += struct.pack("<Q", len(tape))
        for (k, t, c, v) in tape:
            b += struct.pack("<QIIQ", k, t, c, v)
    return bytes(b)


def decode_header(buf):
    assert buf[:8] == MAGIC
    ver, n, num_sms, sm_thr = struct.unpack_from("<IIII", buf, 8)
    dur_thr, flags, hp = struct.unpack_from("<QIi", buf, 24)
    prios = list(struct.unpack_from("<16I", buf, 40))[:n]
    (k_end,) = struct.unpack_from("<Q", buf, 104)
    n_ops = list(struct.unpack_from("<16Q", buf, 112))[:n]
    off = HDR_BYTES
    ops = []
    for c in range(n):
        cl = []
        for _ in range(n_ops[c]):
            kid, kind, opf, cls, sm, _pad, dur = struct.unpack_from("<IHBBIIQ", buf, off)
            cl.append((kid, kind, opf, cls, sm, dur))
            off += 24
        ops.append(cl)
    return dict(version=ver, n_clients=n, num_sms=num_sms, sm_thr=sm_thr, dur_thr=dur_thr,
                flags=flags, hp=hp, prios=prios, k_end=k_end, ops=ops), off


def split_log(buf):
    """Split a full log into (header+ops+tape bytes, tape list, decision-section bytes)."""
    hdr, off = decode_header(buf)
    (nt,) = struct.unpack_from("<Q", buf, off)
    tape = [struct.unpack_from("<QIIQ", buf, off + 8 + 24 * i) for i in range(nt)]
    end = off + 8 + 24 * nt
    return hdr, buf[:end], tape, buf[end:]


def decode_decisions(buf):
    (n,) = struct.unpack_from("<Q", buf, 0)
    out = []
    for i in range(n):
        k, kind, client, _r, kid, seq, be_dur = struct.unpack_from("<QBBHIQq", buf, 8 + 32 * i)
        out.append((k, kind, client, kid, seq, be_dur))
    return out


def parse_golden(path):
    """Parse a tests/golden/we*.txt worked example."""
    cfg = {}
    clients, names = [], {}
    ops = {}
    kid_of = {}
    tape, expect = [], []
    k_end = 0
    for line in open(path):
        line = line.split("#", 1)[0].strip()
        if not line:
            continue
        w = line.split()
        if w[0] == "config":
            for kv in w[1:]:
                key, v = kv.split("=")
                cfg[key] = int(v)
        elif w[0] == "client":
            names[w[1]] = len(clients)
            clients.append(0 if w[2] == "hp" else 1)
            ops[w[1]] = []
        elif w[0] == "op":
            cname, oname, cls, sm, dur = w[1], w[2], w[3], int(w[4]), int(w[5])
            # optional request marks (HP_BUSY_REQUEST): REQ_BEGIN, REQ_END or REQ_BEGIN|REQ_END
            opf = 0
            for m in (w[6].split("|") if len(w) > 6 else []):
                opf |= {"REQ_BEGIN": 1, "REQ_END": 2}[m]
            kid = kid_of.setdefault(oname, len(kid_of) + 1)
            if cls in ("MEMCPY",):
                ops[cname].append((kid, KIND["MEMCPY"], opf, 0, 0, 0))
            else:
                ops[cname].append((kid, 0, opf, CLS[cls], sm, dur))
        elif w[0] == "tape":
            tape.append((int(w[1]), T_VIS if w[2] == "VIS" else T_DONE, names[w[3]], int(w[4])))
        elif w[0] == "kend":
            k_end = int(w[1])
        elif w[0] == "expect":
            k, kind, cname, seq, oname, be_dur = w[1:7]
            expect.append((int(k), DEC_CODES[kind], names[cname],
                           0xFFFFFFFF if oname == "-" else kid_of[oname],
                           (1 << 64) - 1 if seq == "-" else int(seq), int(be_dur)))
    client_ops = [ops[n] for n in sorted(names, key=lambda x: names[x])]
    log = encode(cfg["num_sms"], cfg["sm_thr"], cfg["dur_thr"], cfg["flags"], clients, client_ops,
                 tape, k_end)
    return log, expect
