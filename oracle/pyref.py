"""Pure-Python Gustavson (Alg. 1, L33-50) for tiny inputs -- TEST INFRASTRUCTURE ONLY.

A third, independent transcription used to cross-check `oracle/oracle.c` on small
cases: each C row is a Python dict keyed by column (Alg. 1 lines 6-10), emitted in
sorted column order (§II-B).  fp64 arithmetic in Alg. 1 order, so its values are
bit-identical to oracle.spgemm(method="spa")'s `val`.
"""
from __future__ import annotations


def gustavson(A, B):
    """Return (row_ptr, col, val) lists for C = A x B."""
    rp, col, val = [0], [], []
    for i in range(A.nrows):                                    # line 2
        row = {}
        for p in range(int(A.row_ptr[i]), int(A.row_ptr[i + 1])):  # line 3
            k = int(A.col[p])
            a = float(A.val[p])
            for q in range(int(B.row_ptr[k]), int(B.row_ptr[k + 1])):  # line 4
                j = int(B.col[q])
                value = a * float(B.val[q])                      # line 5
                if j not in row:                                 # line 6
                    row[j] = value                               # lines 7-8
                else:
                    row[j] = row[j] + value                      # line 10
        for j in sorted(row):
            col.append(j)
            val.append(row[j])
        rp.append(len(col))
    return rp, col, val
