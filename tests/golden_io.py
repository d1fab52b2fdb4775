"""Readers for the tiny text fixtures under tests/golden/ (each cites its source)."""
import os

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _lines(name):
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                key, _, val = line.partition(":")
                yield key.strip(), val.split()


def table1_select():
    d = dict(_lines("table1_select.txt"))
    return ([int(v) for v in d["input"]], [(d["pred"][0], int(d["pred"][1]))],
            [int(v) for v in d["output"]])


def q1_worked_example():
    cutoff, rows, expect = None, [], []
    for key, v in _lines("q1_worked_example.txt"):
        if key == "cutoff":
            cutoff = int(v[0])
        elif key == "row":
            rows.append((int(v[0]), v[1], v[2], int(v[3]), int(v[4]), int(v[5]), int(v[6])))
        elif key == "expect":
            expect.append({
                "returnflag": v[0], "linestatus": v[1], "count_order": int(v[2]),
                "sum_qty": int(v[3]), "sum_base_price": int(v[4]), "sum_disc_price": int(v[5]),
                "sum_charge": int(v[6]), "sum_disc": int(v[7]),
                "avg_qty": float(v[8]), "avg_price": float(v[9]), "avg_disc": float(v[10]),
            })
    return cutoff, rows, expect


def rows_to_columns(rows):
    import numpy as np
    return {
        "shipdate": np.array([r[0] for r in rows], dtype=np.int32),
        "returnflag": np.array([ord(r[1]) for r in rows], dtype=np.uint8),
        "linestatus": np.array([ord(r[2]) for r in rows], dtype=np.uint8),
        "quantity": np.array([r[3] for r in rows], dtype=np.int64),
        "extendedprice": np.array([r[4] for r in rows], dtype=np.int64),
        "discount": np.array([r[5] for r in rows], dtype=np.int64),
        "tax": np.array([r[6] for r in rows], dtype=np.int64),
    }


def table1_tuples():
    """Table I's relation as three int32 columns, with its PROJECT and SELECT results."""
    d = dict(_lines("table1_tuples.txt"))
    cols = [[int(v) for v in d[f"field{j}"]] for j in range(3)]
    sel = (d["select_pred"][0], int(d["select_pred"][1]))
    sel_out = tuple(int(v) for v in d["select_out"])
    proj_fields = [int(v) for v in d["project_fields"]]
    po = [int(v) for v in d["project_out"]]
    proj_out = [tuple(po[i:i + len(proj_fields)]) for i in range(0, len(po), len(proj_fields))]
    return cols, sel, sel_out, proj_fields, proj_out
