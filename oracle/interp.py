"""Plain evaluator of an arbitrary stencil spec -- TEST INFRASTRUCTURE ONLY.

The oracle for NEXT-4 (code-generated kernels of unregistered DAGs).  It is
the plain definition of SURVEY 8(c) c1 written out, independent of the C++
front-end (its own tokenizer and recursive-descent parser, no shared code):

  * the DSL subset of the paper's Listing 1: ``parameter``,
    ``iterator``, ``double`` declarations, ``copyin``/``copyout`` (ignored),
    ``#pragma`` / ``#assign`` lines (ignored), one ``stencil NAME(formals)
    {...}`` function and an optional call binding actuals positionally;
  * statements ``double t = e;``, ``t = e;`` and ``X[k][j][i] = e;``;
    expressions with + - * / (C precedence, left associative), unary minus,
    parentheses, numeric literals (correctly rounded by Python's float, as
    strtod), scalars, temporaries, 3D loads ``X[k+a][j+b][i+c]`` and 1D loads
    ``s[i+c]``;
  * radius R per axis = max |offset| over all reads (3D and 1D); interior
    [R, n-R) per axis; every interior point evaluated independently in program
    order (reading R1, R2, R15, R18);
  * a read of an array already written in this function (offset 0) sees the new
    value; an inout array read before its write sees the input (reading R3/R20);
  * IEEE binary64, no contraction (numpy elementwise ops), vectorised over the
    interior: each expression node is an array over all interior points.

``absmode=True`` evaluates the abs-mode DAG of the error gate (reading R13):
every input, scalar and literal replaced by its absolute value and every
``-`` (binary or unary) by ``+``.
"""
from __future__ import annotations

import re

import numpy as np

_TOK = re.compile(r"\s*(?:(\d+\.\d*(?:[eE][+-]?\d+)?|\.\d+(?:[eE][+-]?\d+)?|\d+(?:[eE][+-]?\d+)?)|"
                  r"([A-Za-z_]\w*)|(.))")


def _strip(text):
    text = re.sub(r"/\*.*?\*/", " ", text, flags=re.S)
    lines = []
    for ln in text.splitlines():
        ln = ln.split("//", 1)[0]
        if ln.strip().startswith("#"):
            ln = ""
        lines.append(ln)
    return "\n".join(lines)


def _tokens(text):
    out = []
    for m in _TOK.finditer(text):
        num, ident, op = m.groups()
        if num is not None:
            out.append(("num", num))
        elif ident is not None:
            out.append(("id", ident))
        elif op is not None and not op.isspace():
            out.append(("op", op))
    return out


class Spec:
    """Parsed spec: iterators, declarations, formals, statements (as trees)."""

    def __init__(self, text):
        self.toks = _tokens(_strip(text))
        self.p = 0
        self.iterators = []
        self.decl = {}  # name -> number of dims (0 = scalar)
        self.formals = []
        self.actuals = None
        self.stmts = []
        self.name = None
        self._parse()

    # -- token helpers --
    def peek(self, k=0):
        return self.toks[self.p + k] if self.p + k < len(self.toks) else ("eof", "")

    def take(self, want=None):
        t = self.peek()
        if want is not None and t[1] != want:
            raise SyntaxError(f"expected {want!r}, got {t[1]!r}")
        self.p += 1
        return t

    # -- top level --
    def _parse(self):
        while self.peek()[0] != "eof":
            kind, v = self.peek()
            if v in ("parameter", "copyin", "copyout"):
                while self.take()[1] != ";":
                    pass
            elif v == "iterator":
                self.take()
                while True:
                    self.iterators.append(self.take()[1])
                    if self.take()[1] == ";":
                        break
            elif v == "double":
                self.take()
                while True:
                    name = self.take()[1]
                    nd = 0  # number of extents: "[L,M,N]" or "[L][M][N]" -> 3
                    while self.peek()[1] == "[":
                        self.take()
                        nd += 1
                        depth = 1
                        while depth:
                            t = self.take()[1]
                            depth += (t == "[") - (t == "]")
                            nd += (t == "," and depth == 1)
                    self.decl[name] = nd
                    if self.take()[1] == ";":
                        break
            elif v == "stencil":
                self._stencil()
            elif kind == "id" and self.peek(1)[1] == "(" and v == self.name:
                self.take()
                self.take("(")
                acts = []
                while self.peek()[1] != ")":
                    acts.append(self.take()[1])
                    if self.peek()[1] == ",":
                        self.take()
                self.take(")")
                self.take(";")
                self.actuals = acts
            else:
                raise SyntaxError(f"unexpected token {v!r}")

    def _stencil(self):
        self.take("stencil")
        self.name = self.take()[1]
        self.take("(")
        while self.peek()[1] != ")":
            self.formals.append(self.take()[1])
            if self.peek()[1] == ",":
                self.take()
        self.take(")")
        self.take("{")
        while self.peek()[1] != "}":
            self.stmts.append(self._statement())
        self.take("}")

    def _statement(self):
        declares = False
        if self.peek()[1] == "double":
            self.take()
            declares = True
        name = self.take()[1]
        idx = []
        while self.peek()[1] == "[":
            self.take()
            idx.append(self._index())
            self.take("]")
        self.take("=")
        e = self._expr()
        self.take(";")
        if idx and any(off for _, off in idx):
            raise ValueError("array writes must be at offset 0")
        return ("array" if idx else "temp", name, e, declares)

    def _index(self):
        it = self.take()[1]
        off = 0
        while self.peek()[1] in "+-":
            sgn = 1 if self.take()[1] == "+" else -1
            off += sgn * int(self.take()[1])
        return it, off

    # expression grammar: E = T {(+|-) T}; T = U {(*|/) U}; U = -U | P
    def _expr(self):
        e = self._term()
        while self.peek()[1] in ("+", "-"):
            op = self.take()[1]
            e = (op, e, self._term())
        return e

    def _term(self):
        e = self._unary()
        while self.peek()[1] in ("*", "/"):
            op = self.take()[1]
            e = (op, e, self._unary())
        return e

    def _unary(self):
        if self.peek()[1] == "-":
            self.take()
            return ("neg", self._unary())
        if self.peek()[1] == "+":
            self.take()
            return self._unary()
        return self._primary()

    def _primary(self):
        kind, v = self.take()
        if v == "(":
            e = self._expr()
            self.take(")")
            return e
        if kind == "num":
            return ("num", float(v))
        if self.peek()[1] == "[":
            idx = []
            while self.peek()[1] == "[":
                self.take()
                idx.append(self._index())
                self.take("]")
            return ("load", v, tuple(idx))
        return ("name", v)


def _bind(spec):
    """formal name -> declared (actual) name."""
    acts = spec.actuals if spec.actuals is not None else spec.formals
    if len(acts) != len(spec.formals):
        raise ValueError("call arity differs from the stencil's formals")
    return dict(zip(spec.formals, acts))


def radius(spec):
    """Per-axis radius (z, y, x) over all 3D and 1D reads."""
    its = spec.iterators
    nit = len(its)
    R = [0, 0, 0]

    def walk(e):
        if e[0] == "load":
            for it, off in e[2]:
                ax = 3 - nit + its.index(it)
                R[ax] = max(R[ax], abs(off))
        elif e[0] in ("+", "-", "*", "/"):
            walk(e[1])
            walk(e[2])
        elif e[0] == "neg":
            walk(e[1])

    for st in spec.stmts:
        walk(st[2])
    return tuple(R)


def evaluate(text, dims, arrays, scalars, absmode=False):
    """Evaluate spec `text` on grids of shape `dims` (nz, ny, nx).

    arrays : dict formal name -> numpy array (3D grids: `dims`; 1D: its axis extent)
    scalars: dict formal name -> float
    Returns a dict formal name -> result array for every written grid (copies of
    the input outside the interior; outputs not given as input start as zeros).
    """
    spec = Spec(text)
    bind = _bind(spec)
    its = spec.iterators
    nit = len(its)
    dims = tuple(int(d) for d in dims)
    R = radius(spec)
    lo = [R[a] for a in range(3)]
    hi = [dims[a] - R[a] for a in range(3)]
    if any(h <= l for l, h in zip(lo, hi)):
        raise ValueError("no interior")
    shape = tuple(h - l for l, h in zip(lo, hi))
    A = (lambda x: np.abs(x)) if absmode else (lambda x: x)

    def grid(name):
        g = np.asarray(arrays[name], dtype=np.float64)
        return g.reshape(dims) if g.size == np.prod(dims) else g

    cur = {}  # written grids: current interior values
    temps = {}

    def ev(e):
        k = e[0]
        if k == "num":
            return np.float64(abs(e[1]) if absmode else e[1])
        if k == "name":
            n = e[1]
            if n in temps:
                return temps[n]
            if n in scalars:
                return np.float64(A(scalars[n]))
            raise KeyError(f"unknown name {n}")
        if k == "load":
            n, idx = e[1], e[2]
            if len(idx) == 1 and nit > 1:  # a 1D coefficient array along its iterator's axis
                it, off = idx[0]
                ax = 3 - nit + its.index(it)
                s = np.asarray(arrays[n], dtype=np.float64)
                v = A(s[lo[ax] + off:hi[ax] + off])
                bshape = [1, 1, 1]
                bshape[ax] = shape[ax]
                return np.broadcast_to(v.reshape(bshape), shape)
            offs = [0, 0, 0]
            for it, off in idx:
                offs[3 - nit + its.index(it)] = off
            if n in cur:
                if any(offs):
                    raise ValueError("shifted read of a written array")
                return cur[n]
            g = grid(n)
            sl = tuple(slice(lo[a] + offs[a], hi[a] + offs[a]) for a in range(3))
            return A(g[sl])
        if k == "neg":
            v = ev(e[1])
            return v if absmode else -v
        a, b = ev(e[1]), ev(e[2])
        if k == "+":
            return a + b
        if k == "-":
            return a + b if absmode else a - b
        if k == "*":
            return a * b
        if k == "/":
            return a / b
        raise ValueError(k)

    for kind, name, e, _ in spec.stmts:
        v = np.array(np.broadcast_to(ev(e), shape), dtype=np.float64)
        if kind == "array":
            cur[name] = v
        else:
            temps[name] = v
    out = {}
    for name, v in cur.items():
        base = np.array(grid(name), dtype=np.float64, copy=True) if name in arrays else np.zeros(dims)
        base = base.reshape(dims)
        base[lo[0]:hi[0], lo[1]:hi[1], lo[2]:hi[2]] = v
        out[name] = base
    return out


def formals(text):
    """(formal names, kind per formal: '3d', '1d' or 'scalar', axis of 1D formals)."""
    spec = Spec(text)
    bind = _bind(spec)
    its = spec.iterators
    nit = len(its)
    kinds, axes = {}, {}

    def walk(e):
        if e[0] == "load":
            if len(e[2]) == 1 and nit > 1:
                kinds[e[1]] = "1d"
                axes[e[1]] = 3 - nit + its.index(e[2][0][0])
            else:
                kinds[e[1]] = "3d"
        elif e[0] in ("+", "-", "*", "/"):
            walk(e[1])
            walk(e[2])
        elif e[0] == "neg":
            walk(e[1])

    for kind, name, e, _ in spec.stmts:
        walk(e)
        if kind == "array":
            kinds[name] = "3d"
    out = []
    for f in spec.formals:
        nd = spec.decl.get(bind[f], None)
        if f in kinds:
            out.append((f, kinds[f], axes.get(f)))
        elif nd == 0:
            out.append((f, "scalar", None))
        else:
            out.append((f, "3d" if nd != 1 else "1d", None))
    return out


def roles(text):
    """3D formal -> 'in' | 'out' | 'inout' (written and read before the write)."""
    spec = Spec(text)
    nit = len(spec.iterators)
    written, read_before, read = set(), set(), set()

    def walk(e):
        if e[0] == "load" and not (len(e[2]) == 1 and nit > 1):
            read.add(e[1])
            if e[1] not in written:
                read_before.add(e[1])
        elif e[0] in ("+", "-", "*", "/"):
            walk(e[1])
            walk(e[2])
        elif e[0] == "neg":
            walk(e[1])

    for kind, name, e, _ in spec.stmts:
        walk(e)
        if kind == "array":
            written.add(name)
    out = {}
    for f, k, _ in formals(text):
        if k != "3d":
            continue
        out[f] = ("inout" if f in read_before else "out") if f in written else "in"
    return out


# ---------------------------------------------------------------------------
# Multi-stencil programs (Fig 3c): several stencil
# definitions and calls in sequence.  The plain definition: the calls run in
# program order, each one a complete evaluation of its stencil (above) on the
# arrays as the previous calls left them; a call's written grids replace the
# bound arrays' interiors.  Programs take declared names (not formals).
# ---------------------------------------------------------------------------

def _split_program(text):
    """-> (prelude text, {stencil name: definition text}, [(name, call text)])"""
    t = _strip(text)
    defs, calls, prelude = {}, [], []
    i = 0
    stmt_start = 0
    while i < len(t):
        m = re.match(r"\s*stencil\s+([A-Za-z_]\w*)", t[i:])
        if m and (i == 0 or not (t[i - 1].isalnum() or t[i - 1] == "_")) and t[i:i + m.end()].strip().startswith("stencil"):
            j = t.index("{", i)
            depth, k = 0, j
            while True:
                depth += (t[k] == "{") - (t[k] == "}")
                k += 1
                if depth == 0:
                    break
            defs[m.group(1)] = t[i:k]
            i = k
            stmt_start = i
            continue
        if t[i] == ";":
            stmt = t[stmt_start:i + 1]
            cm = re.match(r"\s*([A-Za-z_]\w*)\s*\(", stmt)
            if cm and cm.group(1) in defs:
                calls.append((cm.group(1), stmt))
            else:
                prelude.append(stmt)
            stmt_start = i + 1
        i += 1
    return "\n".join(prelude), defs, calls


def program_stages(text):
    """[(single-stencil spec text, {formal: declared name})] in call order."""
    prelude, defs, calls = _split_program(text)
    if not calls:
        if len(defs) != 1:
            raise ValueError("several stencils but no call")
        (name, d), = defs.items()
        one = prelude + "\n" + d
        return [(one, {f: f for f in Spec(one).formals})]
    out = []
    for name, c in calls:
        one = prelude + "\n" + defs[name] + "\n" + c
        sp = Spec(one)
        out.append((one, _bind(sp)))
    return out


def evaluate_program(text, dims, arrays, scalars, absmode=False):
    """Evaluate a program; arrays / scalars keyed by DECLARED names.  Returns a
    dict declared name -> grid for every array some stage wrote.  With
    absmode=True every stage runs in abs mode on the abs-mode results of the
    earlier stages (the error-gate bound of the composition, reading R13)."""
    state = {k: np.array(v, dtype=np.float64, copy=True) for k, v in arrays.items()}
    written = set()
    for one, bind in program_stages(text):
        fa = {f: state[a] for f, a in bind.items() if a in state}
        fs = {f: scalars[a] for f, a in bind.items() if a in scalars}
        res = evaluate(one, dims, fa, fs, absmode=absmode)
        for f, g in res.items():
            state[bind[f]] = g
            written.add(bind[f])
    return {k: state[k] for k in written}
