"""memcached binary-protocol GET over UDP, as a plain definition -- TEST INFRASTRUCTURE ONLY.

Config 4 (sec. VIII-D: "a binary UDP memcached version ... the GPU supports only
GETs"): for a request datagram (8-byte UDP frame header + 24-byte binary request header + key),
the reply is the frame header echoing the request id (sequence 0, 1 datagram), then a binary
response header (magic 0x81, opcode echoed, key length 0, CAS 0, opaque echoed) with either
status 0, 4 bytes of flags (0) and the stored value, or status 1 and "Not found".  The key/value
store is a Python dict -- no hashing, bucketing or layout shared with the CUDA path.
"""
from __future__ import annotations

import struct


def expected_response(packet: bytes, table: dict) -> bytes | None:
    if len(packet) < 32 or packet[8] != 0x80 or packet[9] != 0x00:
        return None                                   # malformed: the server sends nothing
    req_id = packet[0:2]
    _, opcode, klen, ext, _, _, body, opaque, _ = struct.unpack(">BBHBBHIIQ", packet[8:32])
    if klen < 1 or klen > 32 or 32 + ext + klen > len(packet):
        return None
    key = packet[32 + ext: 32 + ext + klen]
    frame = req_id + struct.pack(">HHH", 0, 1, 0)
    if key in table:
        v = table[key]
        hdr = struct.pack(">BBHBBHIIQ", 0x81, opcode, 0, 4, 0, 0, 4 + len(v), opaque, 0)
        return frame + hdr + b"\0\0\0\0" + v
    hdr = struct.pack(">BBHBBHIIQ", 0x81, opcode, 0, 0, 0, 1, 9, opaque, 0)
    return frame + hdr + b"Not found"
