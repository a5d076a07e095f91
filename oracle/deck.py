"""CloverLeaf text decks <-> workloads deck dicts.

TEST INFRASTRUCTURE ONLY (like the rest of oracle/).  The oracle's
command-line driver (clover_oracle_main.cpp) reads the reference's
``*clover ... *endclover`` text form; the harness converts a JSON / dict deck
to that form with ``deck_to_text`` and back with ``parse_text_deck``.  No
arithmetic of the method lives here.
"""
from __future__ import annotations

GRID_KEYS = (("x_cells", int), ("y_cells", int), ("xmin", float), ("ymin", float),
             ("xmax", float), ("ymax", float), ("initial_timestep", float),
             ("max_timestep", float), ("timestep_rise", float), ("end_step", int),
             ("advect_x_first", int), ("dtmin", float), ("dtc_safe", float),
             ("dtu_safe", float), ("dtv_safe", float), ("dtdiv_safe", float),
             ("summary_every", int))
STATE_KEYS = ("density", "energy", "xvel", "yvel", "xmin", "xmax", "ymin", "ymax", "radius")
MIRRORS = {0: "geometric", 1: "cellcentre"}


def _num(v) -> str:
    return repr(float(v)) if isinstance(v, float) else str(v)


def deck_to_text(deck: dict) -> str:
    """A workloads-style deck dict as a CloverLeaf text deck (every float
    written with repr(): round-trip exact)."""
    out = ["*clover"]
    for i, s in enumerate(deck["states"], 1):
        parts = [f" state {i}"]
        for k in STATE_KEYS:
            if k in s and (k in ("density", "energy") or s[k] != 0.0):
                parts.append(f"{k}={_num(float(s[k]))}")
        if i > 1:
            parts.append(f"geometry={s.get('geometry', 'rectangle')}")
        out.append(" ".join(parts))
    parts = []
    for k, typ in GRID_KEYS:
        if k in deck:
            parts.append(f"{k}={_num(typ(deck[k]))}")
    out.append(" " + " ".join(parts))
    out.append(f" face_mirror={MIRRORS[int(deck.get('face_mirror', 0))]}")
    out.append("*endclover")
    return "\n".join(out) + "\n"


def parse_text_deck(text: str) -> dict:
    """The inverse of deck_to_text (keys the harness uses)."""
    deck: dict = {"states": []}
    inside = False
    for line in text.splitlines():
        line = line.split("!", 1)[0].strip()
        if not line:
            continue
        low = line.lower()
        if low == "*clover":
            inside = True
            continue
        if low == "*endclover":
            inside = False
            continue
        if not inside:
            continue
        tok = line.split()
        if tok[0].lower() == "state":
            n = int(tok[1])
            while len(deck["states"]) < n:
                deck["states"].append({"geometry": "rectangle", "xvel": 0.0, "yvel": 0.0,
                                       "xmin": 0.0, "xmax": 0.0, "ymin": 0.0, "ymax": 0.0,
                                       "radius": 0.0})
            st = deck["states"][n - 1]
            for t in tok[2:]:
                k, v = t.split("=", 1)
                k = k.lower()
                st[k] = v.lower() if k == "geometry" else float(v)
            continue
        for t in tok:
            k, v = t.split("=", 1)
            k = k.lower()
            if k == "face_mirror":
                deck[k] = {"geometric": 0, "cellcentre": 1}[v.lower()]
                continue
            typ = dict(GRID_KEYS).get(k, float)
            deck[k] = typ(float(v)) if typ is int else float(v)
    return deck
