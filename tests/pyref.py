"""Independent pure-Python references used only to PIN the oracle.

Nothing here is shared with the oracle or the CUDA path: the fingerprint is a
big-integer GF(2) long division of the window polynomial (the plain
definition of SURVEY 8(c) step 1), and chunking is the brute-force greedy
definition over that fingerprint.
"""
POLY = 0x45C2B6A1
WINDOW = 32


def gf2_mod(x: int, poly: int = POLY) -> int:
    """x(t) mod P(t), P(t) = t^32 + poly, by long division over GF(2)."""
    P = (1 << 32) | poly
    while x.bit_length() > 32:
        x ^= P << (x.bit_length() - 33)
    return x


def fp(window: bytes, poly: int = POLY) -> int:
    # earlier bytes are the higher-degree coefficients, MSB first (reading O4)
    return gf2_mod(int.from_bytes(bytes(window), "big"), poly)


def chunk_bruteforce(data: bytes, mask=0xFFF, value=0, window=WINDOW, min_chunk=WINDOW,
                     max_chunk=0, poly=POLY):
    """Greedy definition: next cut = smallest e >= c+min_chunk (e < n) with
    (fp(data[e-window:e]) & mask) == value, or c+max_chunk; item end closes."""
    n = len(data)
    cand = [False] * (n + 1)
    for e in range(window, n):
        cand[e] = (fp(data[e - window:e], poly) & mask) == value
    starts, c = [], 0
    while c < n:
        starts.append(c)
        e = n
        for x in range(c + 1, n):
            if max_chunk and x - c >= max_chunk:
                e = x
                break
            if x - c >= max(min_chunk, window) and cand[x]:
                e = x
                break
        c = e
    return starts


def literal_fp(seg: bytes, poly: int = POLY, window: int = WINDOW) -> int:
    """PARSEC's hash with the window table of length 0 (reading O5-L) after
    reading seg = data[c:n] from a restart at c, as a closed form: every byte
    p[k] enters at degree 8 (n - 1 - k), and every byte with k <= n - 1 -
    window is XORed in once more when it leaves the window, then shifted
    n - window - k times:  h = sum_k p[k] t^{8(n-1-k)} + sum_{k <= n-1-window}
    p[k] t^{8(n-window-k)}  (mod P), by big-integer long division."""
    n = len(seg)
    x = 0
    for k, b in enumerate(seg):
        x ^= b << (8 * (n - 1 - k))
        if k <= n - 1 - window:
            x ^= b << (8 * (n - window - k))
    return gf2_mod(x, poly)


def chunk_bruteforce_literal(data: bytes, mask=0xFFF, value=0, window=WINDOW, poly=POLY):
    """Greedy definition for the literal mode: from a cut c, the next cut is
    the smallest e >= c + window (e < n) with (literal_fp(data[c:e]) & mask)
    == value; the item end closes the last chunk."""
    n = len(data)
    starts, c = [], 0
    while c < n:
        starts.append(c)
        e = n
        for x in range(c + window, n):
            if (literal_fp(data[c:x], poly, window) & mask) == value:
                e = x
                break
        c = e
    return starts
