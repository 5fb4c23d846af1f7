"""Task function ids and argument-block layouts of include/pagoda_tasks.h, as
numpy structured dtypes (one record = one task's inline args, <= 40 bytes).

Marshalling only: these are the byte layouts the C structs have.
"""
import numpy as np

NOP, MARK, TID, BAR, SMEM, SPIN, GATE, HOLD, PAPER = 0, 1, 2, 3, 4, 5, 6, 7, 8
MB, TDES, MM, FB, BF, CONV, DCT = 16, 17, 18, 19, 20, 21, 22
MM_TC = 23
MM64 = 24   # Table 4's 64x64 MatrixMul (NEXT-4)

NAMES = {NOP: "nop", MARK: "mark", TID: "tid", BAR: "bar", SMEM: "smem", SPIN: "spin", GATE: "gate",
         HOLD: "hold", PAPER: "paper",
         MB: "mb", TDES: "tdes", MM: "mm", FB: "fb", BF: "bf", CONV: "conv", DCT: "dct", MM_TC: "mm_tc", MM64: "mm64"}

_p = "<u8"
ARGS = {
    MARK: np.dtype([("out", _p), ("cnt", _p), ("base", "<u4"), ("tag", "<u4")]),
    TID: np.dtype([("out", _p), ("base", "<u4"), ("pad", "<u4")]),
    BAR: np.dtype([("err", _p), ("scratch", _p), ("phases", "<u4"), ("pad", "<u4")]),
    SMEM: np.dtype([("err", _p), ("bytes", "<u4"), ("spin_ns", "<u4"), ("seed", "<u4"), ("pad", "<u4")]),
    SPIN: np.dtype([("ns", "<u8")]),
    GATE: np.dtype([("flag", _p)]),
    HOLD: np.dtype([("flag", _p), ("err", _p), ("started", _p), ("seed", "<u4"), ("pad", "<u4")]),
    PAPER: np.dtype([("out", _p), ("err", _p), ("base", "<u4"), ("pad", "<u4")]),
    MB: np.dtype([("out", _p), ("x0", "<f4"), ("y0", "<f4"), ("dx", "<f4"), ("tx", "<i4"), ("ty", "<i4"),
                  ("maxit", "<i4")]),
    TDES: np.dtype([("inp", _p), ("out", _p), ("tables", _p), ("nblk", "<u4"), ("pad", "<u4")]),
    MM: np.dtype([("A", _p), ("B", _p), ("C", _p)]),
    MM_TC: np.dtype([("A", _p), ("B", _p), ("C", _p)]),
    MM64: np.dtype([("A", _p), ("B", _p), ("C", _p)]),
    FB: np.dtype([("r", _p), ("H", _p), ("F", _p), ("y", _p), ("scratch", _p)]),
    BF: np.dtype([("x", _p), ("h", _p), ("w", _p), ("out", _p)]),
    CONV: np.dtype([("img", _p), ("krow", _p), ("kcol", _p), ("out", _p), ("scratch", _p)]),
    DCT: np.dtype([("img", _p), ("coef", _p), ("out", _p)]),
}
for _k, _d in ARGS.items():
    assert _d.itemsize <= 40, (_k, _d.itemsize)

# a generic 40-byte arg record (heterogeneous spawns: one row per task)
RAW = np.dtype([("b", "u1", (40,))])


def records(func_id: int, n: int) -> np.ndarray:
    return np.zeros(n, ARGS[func_id])


def to_raw(rec: np.ndarray) -> np.ndarray:
    """Copy structured args into 40-byte rows (for mixed-body spawns)."""
    out = np.zeros((len(rec), 40), np.uint8)
    out[:, :rec.dtype.itemsize] = rec.view(np.uint8).reshape(len(rec), rec.dtype.itemsize)
    return out


TDES_TABLE_BYTES = 2048 + 384 + 16384 + 16384
