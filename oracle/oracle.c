/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct CPU oracle for multi-pattern regex
 * matching with all-match, match-END semantics.  Only tests/, bench.py's
 * cpu_baseline / --impl reference leg and __graft_entry__.smoke() may load it.
 * It shares no code (no parser, no tables, no helpers) with the CUDA path in
 * paper_conf_micro_ge0025_b200/.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, "P:Lnnn" = its line):
 *   S_r[i] = 1  <=>  there is s <= i with input[s..i] in L(r)
 *   (non-empty matches, unanchored, byte alphabet).  This is the paper's
 *   definition of the match bitstream S_R "such that a 1 at position i
 *   indicates a successful match ending at that position", under all-match
 *   semantics (Sec. 2 "Lowering Regular Expressions ..."); grammar of
 *   P:L67-69 (CC, RR, R|R, R*, R{n,m}, R+, R?); counts and positions are what
 *   the paper validates.  Readings where the paper is silent are
 *   listed in DESIGN.md Sec. "Readings" (c1..c17 of SURVEY.md Sec. 8(c)):
 *   non-empty matches only (c1), 0-based offset of the last byte (c2),
 *   unanchored (c3), '.' = any byte but '\n', negated classes include '\n',
 *   whole-stream matching (c4), raw bytes, case-sensitive, Python-re escapes
 *   (c5), R{n,m} = R^n (R?)^(m-n) (c7), count = popcount(S_r) (c10).
 *
 * Algorithm: Thompson NFA construction and simulation (Thompson 1968, the
 * paper's ref [75]; the automata view of P:L71).  For every input
 * byte i (P:L120 positions), the start closure is injected BEFORE stepping
 * (unanchored), the byte is consumed, and S[i] = 1 iff the MATCH state is in
 * the resulting closure.  MATCH is tested only after a byte is consumed, so
 * the empty match is never reported.
 *
 * Optional memoisation (RE2-style lazy DFA, the paper's ref [5]):
 * key = set of NFA states (bitset) -> DFA id, transitions filled lazily;
 * bounded, flushed when full.  tests/ check that it equals the uncached run.
 *
 * Digests (for parity at sizes where dense streams do not fit): additive
 * mod 2^64 sums d1 = sum splitmix64(p), d2 = sum splitmix64(p ^ 0x9E37..15)
 * over the match-end positions p.
 */
#include <pthread.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------ */
/* byte sets                                                           */
/* ------------------------------------------------------------------ */
typedef struct { uint64_t w[4]; } bset;

static void bs_clear(bset *s) { memset(s, 0, sizeof *s); }
static void bs_add(bset *s, int c) { s->w[c >> 6] |= 1ull << (c & 63); }
static int bs_has(const bset *s, int c) { return (int)((s->w[c >> 6] >> (c & 63)) & 1); }
static void bs_add_range(bset *s, int a, int b) { for (int c = a; c <= b; c++) bs_add(s, c); }
static void bs_or(bset *d, const bset *s) { for (int i = 0; i < 4; i++) d->w[i] |= s->w[i]; }
static void bs_not(bset *s) { for (int i = 0; i < 4; i++) s->w[i] = ~s->w[i]; }

/* Python-re (bytes) meanings of \d \w \s (c5) */
static void bs_digit(bset *s) { bs_add_range(s, '0', '9'); }
static void bs_word(bset *s) {
  bs_add_range(s, 'a', 'z'); bs_add_range(s, 'A', 'Z'); bs_add_range(s, '0', '9'); bs_add(s, '_');
}
static void bs_space(bset *s) {
  bs_add(s, ' '); bs_add(s, '\t'); bs_add(s, '\n'); bs_add(s, '\r'); bs_add(s, '\f'); bs_add(s, '\v');
}

/* ------------------------------------------------------------------ */
/* AST                                                                 */
/* ------------------------------------------------------------------ */
enum { A_EMPTY, A_SET, A_CAT, A_ALT, A_STAR, A_PLUS, A_QUEST, A_REP };
typedef struct ast {
  int kind;
  bset set;
  struct ast *a, *b;
  int lo, hi; /* A_REP: hi = -1 means unbounded */
} ast;

typedef struct {
  const unsigned char *p;
  size_t n, i;
  int err;        /* 0 ok, 1 parse error, 2 unsupported, 3 too big */
  size_t err_at;
  char msg[160];
  ast **pool;
  size_t npool, cap;
} parser;

static ast *mk(parser *ps, int kind) {
  if (ps->npool == ps->cap) {
    ps->cap = ps->cap ? 2 * ps->cap : 64;
    ps->pool = (ast **)realloc(ps->pool, ps->cap * sizeof(ast *));
  }
  ast *x = (ast *)calloc(1, sizeof(ast));
  x->kind = kind;
  ps->pool[ps->npool++] = x;
  return x;
}

static void fail(parser *ps, int code, const char *m) {
  if (!ps->err) {
    ps->err = code;
    ps->err_at = ps->i;
    snprintf(ps->msg, sizeof ps->msg, "%s", m);
  }
}

static int peek(parser *ps) { return ps->i < ps->n ? ps->p[ps->i] : -1; }

static int hexval(int c) {
  if (c >= '0' && c <= '9') return c - '0';
  if (c >= 'a' && c <= 'f') return c - 'a' + 10;
  if (c >= 'A' && c <= 'F') return c - 'A' + 10;
  return -1;
}

/* Parse an escape after '\'.  Sets *single to the byte (if a single byte)
 * or fills *set (for \d \w \s and negations).  Returns 1 for single, 2 for
 * set, 0 on error. */
static int parse_escape(parser *ps, int *single, bset *set, int in_class) {
  int c = peek(ps);
  if (c < 0) { fail(ps, 1, "trailing backslash"); return 0; }
  ps->i++;
  switch (c) {
    case 'n': *single = '\n'; return 1;
    case 'r': *single = '\r'; return 1;
    case 't': *single = '\t'; return 1;
    case 'f': *single = '\f'; return 1;
    case 'v': *single = '\v'; return 1;
    case 'a': *single = 7; return 1;
    case 'x': {
      int h1 = ps->i < ps->n ? hexval(ps->p[ps->i]) : -1;
      int h2 = ps->i + 1 < ps->n ? hexval(ps->p[ps->i + 1]) : -1;
      if (h1 < 0 || h2 < 0) { fail(ps, 1, "bad \\x escape"); return 0; }
      ps->i += 2;
      *single = h1 * 16 + h2;
      return 1;
    }
    case 'd': case 'D': case 'w': case 'W': case 's': case 'S':
      bs_clear(set);
      if (c == 'd' || c == 'D') bs_digit(set);
      if (c == 'w' || c == 'W') bs_word(set);
      if (c == 's' || c == 'S') bs_space(set);
      if (c == 'D' || c == 'W' || c == 'S') bs_not(set);
      return 2;
    case 'b': case 'B': case 'A': case 'Z':
      (void)in_class;
      fail(ps, 2, "anchors / word boundaries are unsupported");
      return 0;
    default:
      if ((c >= 'a' && c <= 'z') || (c >= 'A' && c <= 'Z') || (c >= '0' && c <= '9')) {
        fail(ps, (c >= '0' && c <= '9') ? 2 : 1, "unknown or unsupported escape");
        return 0;
      }
      *single = c; /* escaped punctuation / space / high byte: the byte itself */
      return 1;
  }
}

static ast *parse_alt(parser *ps);

static ast *parse_class(parser *ps) {
  /* '[' already consumed */
  ast *x = mk(ps, A_SET);
  int neg = 0;
  if (peek(ps) == '^') { neg = 1; ps->i++; }
  int first = 1;
  for (;;) {
    int c = peek(ps);
    if (c < 0) { fail(ps, 1, "unterminated class"); return x; }
    if (c == ']' && !first) { ps->i++; break; }
    first = 0;
    int lo_single = -1;
    bset tmp;
    if (c == '\\') {
      ps->i++;
      int r = parse_escape(ps, &lo_single, &tmp, 1);
      if (!r) return x;
      if (r == 2) { bs_or(&x->set, &tmp); continue; }
    } else {
      lo_single = c;
      ps->i++;
    }
    /* a range? */
    if (peek(ps) == '-' && ps->i + 1 < ps->n && ps->p[ps->i + 1] != ']') {
      ps->i++; /* '-' */
      int hi_single = -1;
      int d = peek(ps);
      if (d == '\\') {
        ps->i++;
        int r = parse_escape(ps, &hi_single, &tmp, 1);
        if (!r) return x;
        if (r == 2) { fail(ps, 1, "bad range"); return x; }
      } else {
        hi_single = d;
        ps->i++;
      }
      if (hi_single < lo_single) { fail(ps, 1, "bad range"); return x; }
      bs_add_range(&x->set, lo_single, hi_single);
    } else {
      bs_add(&x->set, lo_single);
    }
  }
  if (neg) bs_not(&x->set);
  return x;
}

static ast *parse_atom(parser *ps) {
  int c = peek(ps);
  if (c == '(') {
    ps->i++;
    if (peek(ps) == '?') {
      if (ps->i + 1 < ps->n && ps->p[ps->i + 1] == ':') {
        ps->i += 2;
      } else {
        fail(ps, 2, "unsupported group extension");
        return NULL;
      }
    }
    ast *inner = parse_alt(ps);
    if (ps->err) return NULL;
    if (peek(ps) != ')') { fail(ps, 1, "missing )"); return NULL; }
    ps->i++;
    return inner;
  }
  if (c == '[') { ps->i++; return parse_class(ps); }
  if (c == '.') {
    ps->i++;
    ast *x = mk(ps, A_SET);
    bs_add_range(&x->set, 0, 255);
    x->set.w['\n' >> 6] &= ~(1ull << ('\n' & 63)); /* '.' excludes '\n' (c4) */
    return x;
  }
  if (c == '\\') {
    ps->i++;
    int single = -1;
    bset tmp;
    int r = parse_escape(ps, &single, &tmp, 0);
    if (!r) return NULL;
    ast *x = mk(ps, A_SET);
    if (r == 2) x->set = tmp; else bs_add(&x->set, single);
    return x;
  }
  if (c == '^' || c == '$') { fail(ps, 2, "anchors are unsupported"); return NULL; }
  if (c == '*' || c == '+' || c == '?') { fail(ps, 1, "nothing to repeat"); return NULL; }
  if (c == '{') { fail(ps, 1, "nothing to repeat / bare '{'"); return NULL; }
  ps->i++;
  ast *x = mk(ps, A_SET);
  bs_add(&x->set, c);
  return x;
}

static int parse_int(parser *ps, int *v) {
  int got = 0;
  long acc = 0;
  while (ps->i < ps->n && ps->p[ps->i] >= '0' && ps->p[ps->i] <= '9') {
    acc = acc * 10 + (ps->p[ps->i] - '0');
    if (acc > 100000) acc = 100000;
    ps->i++;
    got = 1;
  }
  *v = (int)acc;
  return got;
}

static ast *parse_repeat(parser *ps) {
  ast *x = parse_atom(ps);
  if (ps->err || !x) return x;
  int nq = 0;
  for (;;) {
    int c = peek(ps);
    int kind = -1, lo = 0, hi = 0;
    if (c == '*') { kind = A_STAR; ps->i++; }
    else if (c == '+') { kind = A_PLUS; ps->i++; }
    else if (c == '?') { kind = A_QUEST; ps->i++; }
    else if (c == '{') {
      size_t save = ps->i;
      ps->i++;
      int a = 0, b = 0, ha = parse_int(ps, &a), hb;
      if (peek(ps) == '}') {
        if (!ha) { ps->i = save; fail(ps, 1, "bad {} quantifier"); return x; }
        ps->i++; lo = hi = a;
      } else if (peek(ps) == ',') {
        ps->i++;
        hb = parse_int(ps, &b);
        if (peek(ps) != '}') { ps->i = save; fail(ps, 1, "bad {} quantifier"); return x; }
        ps->i++;
        lo = ha ? a : 0;
        hi = hb ? b : -1;
        if (hi >= 0 && hi < lo) { fail(ps, 1, "min repeat greater than max repeat"); return x; }
      } else {
        ps->i = save;
        fail(ps, 1, "bad {} quantifier");
        return x;
      }
      kind = A_REP;
    } else {
      break;
    }
    if (nq) { fail(ps, (c == '?' || c == '+') ? 2 : 1, "multiple repeat / lazy or possessive quantifier"); return x; }
    nq = 1;
    if (kind == A_REP && (lo > 1000 || hi > 1000)) { fail(ps, 3, "repetition count too large"); return x; }
    ast *q = mk(ps, kind);
    q->a = x;
    q->lo = lo;
    q->hi = hi;
    x = q;
  }
  return x;
}

static ast *parse_cat(parser *ps) {
  ast *x = NULL;
  for (;;) {
    int c = peek(ps);
    if (c < 0 || c == '|' || c == ')') break;
    ast *y = parse_repeat(ps);
    if (ps->err) return NULL;
    if (!x) x = y;
    else {
      ast *k = mk(ps, A_CAT);
      k->a = x;
      k->b = y;
      x = k;
    }
  }
  if (!x) x = mk(ps, A_EMPTY);
  return x;
}

static ast *parse_alt(parser *ps) {
  ast *x = parse_cat(ps);
  while (!ps->err && peek(ps) == '|') {
    ps->i++;
    ast *y = parse_cat(ps);
    if (ps->err) return NULL;
    ast *k = mk(ps, A_ALT);
    k->a = x;
    k->b = y;
    x = k;
  }
  return x;
}

/* ------------------------------------------------------------------ */
/* Thompson NFA                                                        */
/* ------------------------------------------------------------------ */
enum { S_CHAR, S_SPLIT, S_MATCH };
typedef struct {
  int type;
  int out, out1; /* S_SPLIT: two epsilon edges (out1 may be -1 = plain epsilon) */
  bset set;
} nstate;

typedef struct {
  nstate *st;
  int n, cap;
  int too_big;
} nfa_builder;

#define MAX_NFA_STATES 200000

static int new_state(nfa_builder *b, int type, int out, int out1) {
  if (b->n >= MAX_NFA_STATES) { b->too_big = 1; return 0; }
  if (b->n == b->cap) {
    b->cap = b->cap ? 2 * b->cap : 256;
    b->st = (nstate *)realloc(b->st, (size_t)b->cap * sizeof(nstate));
  }
  nstate *s = &b->st[b->n];
  memset(s, 0, sizeof *s);
  s->type = type;
  s->out = out;
  s->out1 = out1;
  return b->n++;
}

/* Build the fragment for x whose exit goes to state `next`; return its entry
 * state.  Built back to front, so every copy of a repeated sub-expression
 * gets fresh states (R{n,m} expansion by copying, c7). */
static int build(nfa_builder *b, const ast *x, int next) {
  if (b->too_big) return next;
  switch (x->kind) {
    case A_EMPTY: return next;
    case A_SET: {
      int s = new_state(b, S_CHAR, next, -1);
      b->st[s].set = x->set;
      return s;
    }
    case A_CAT: {
      int sb = build(b, x->b, next);
      return build(b, x->a, sb);
    }
    case A_ALT: {
      int sa = build(b, x->a, next);
      int sb = build(b, x->b, next);
      return new_state(b, S_SPLIT, sa, sb);
    }
    case A_STAR: { /* loop: SPLIT(body, next); body exits to loop */
      int loop = new_state(b, S_SPLIT, -1, next);
      int body = build(b, x->a, loop);
      b->st[loop].out = body;
      return loop;
    }
    case A_PLUS: { /* body then loop back */
      int loop = new_state(b, S_SPLIT, -1, next);
      int body = build(b, x->a, loop);
      b->st[loop].out = body;
      return body;
    }
    case A_QUEST: {
      int sa = build(b, x->a, next);
      return new_state(b, S_SPLIT, sa, next);
    }
    case A_REP: {
      int tail = next;
      if (x->hi < 0) {
        ast star;
        memset(&star, 0, sizeof star);
        star.kind = A_STAR;
        star.a = x->a;
        tail = build(b, &star, next);
      } else {
        for (int i = 0; i < x->hi - x->lo; i++) {
          int body = build(b, x->a, tail); /* (R (rest)?) nesting = R? R? ... */
          tail = new_state(b, S_SPLIT, body, next);
        }
      }
      for (int i = 0; i < x->lo; i++) tail = build(b, x->a, tail);
      return tail;
    }
  }
  return next;
}

/* ------------------------------------------------------------------ */
/* compiled regex: NFA + closures                                      */
/* ------------------------------------------------------------------ */
typedef struct orc_regex {
  int nst;      /* NFA states */
  int nw;       /* bitset words */
  nstate *st;
  uint64_t *start;    /* closure({q0}) */
  uint64_t *after;    /* per state: closure({out}) for S_CHAR states (nw words each) */
  int match_state;
  int nullable;
  int64_t max_len; /* longest string of L(r), -1 = unbounded (see ast_max_len) */
} orc_regex;

/* Longest string length of L(x) (an upper bound on the length of any match,
 * used by the tests to window the oracle exactly: a match ending at i starts
 * at >= i - max_len + 1); -1 = unbounded.  Straight from the grammar of
 * Sec. 2: concatenation adds, alternation takes the maximum, a
 * repetition multiplies its upper count, an unbounded repetition of a body
 * that can consume a byte is unbounded. */
static int64_t ast_max_len(const ast *x) {
  int64_t a, b;
  switch (x->kind) {
    case A_EMPTY: return 0;
    case A_SET: return 1;
    case A_CAT:
      a = ast_max_len(x->a);
      b = ast_max_len(x->b);
      return (a < 0 || b < 0) ? -1 : a + b;
    case A_ALT:
      a = ast_max_len(x->a);
      b = ast_max_len(x->b);
      return (a < 0 || b < 0) ? -1 : (a > b ? a : b);
    case A_QUEST: return ast_max_len(x->a);
    case A_STAR:
    case A_PLUS:
      a = ast_max_len(x->a);
      return a == 0 ? 0 : -1;
    case A_REP:
      a = ast_max_len(x->a);
      if (a == 0) return 0;
      if (a < 0 || x->hi < 0) return -1;
      return a * (int64_t)x->hi;
  }
  return -1;
}

static void closure_add(const orc_regex *r, int s, uint64_t *set, int *stack) {
  int sp = 0;
  if (s < 0) return;
  stack[sp++] = s;
  while (sp) {
    int q = stack[--sp];
    if (q < 0) continue;
    if ((set[q >> 6] >> (q & 63)) & 1) continue;
    set[q >> 6] |= 1ull << (q & 63);
    if (r->st[q].type == S_SPLIT) {
      if (r->st[q].out >= 0) stack[sp++] = r->st[q].out;
      if (r->st[q].out1 >= 0) stack[sp++] = r->st[q].out1;
    }
  }
}

int orc_compile(const char *pat, size_t len, orc_regex **out, size_t *err_at, char *msg, size_t msglen) {
  parser ps;
  memset(&ps, 0, sizeof ps);
  ps.p = (const unsigned char *)pat;
  ps.n = len;
  ast *root = parse_alt(&ps);
  if (!ps.err && ps.i != ps.n) fail(&ps, 1, "unbalanced parenthesis");
  int code = ps.err;
  if (code) {
    if (err_at) *err_at = ps.err_at;
    if (msg && msglen) snprintf(msg, msglen, "%s", ps.msg);
  } else {
    nfa_builder b;
    memset(&b, 0, sizeof b);
    int m = new_state(&b, S_MATCH, -1, -1);
    int q0 = build(&b, root, m);
    if (b.too_big) {
      code = 3;
      if (err_at) *err_at = 0;
      if (msg && msglen) snprintf(msg, msglen, "expansion too large");
      free(b.st);
    } else {
      orc_regex *r = (orc_regex *)calloc(1, sizeof *r);
      r->nst = b.n;
      r->st = b.st;
      r->nw = (b.n + 63) / 64;
      r->match_state = m;
      r->start = (uint64_t *)calloc((size_t)r->nw, 8);
      r->after = (uint64_t *)calloc((size_t)r->nw * (size_t)r->nst, 8);
      int *stack = (int *)malloc(sizeof(int) * (size_t)(2 * r->nst + 4));
      closure_add(r, q0, r->start, stack);
      for (int s = 0; s < r->nst; s++)
        if (r->st[s].type == S_CHAR) closure_add(r, r->st[s].out, r->after + (size_t)s * r->nw, stack);
      free(stack);
      r->nullable = (int)((r->start[m >> 6] >> (m & 63)) & 1);
      r->max_len = root ? ast_max_len(root) : 0;
      *out = r;
    }
  }
  for (size_t k = 0; k < ps.npool; k++) free(ps.pool[k]);
  free(ps.pool);
  return code;
}

void orc_free(orc_regex *r) {
  if (!r) return;
  free(r->st);
  free(r->start);
  free(r->after);
  free(r);
}

int orc_num_states(const orc_regex *r) { return r->nst; }
int orc_nullable(const orc_regex *r) { return r->nullable; }
int64_t orc_max_len(const orc_regex *r) { return r->max_len; }

/* One NFA step: nxt = closure(delta(src, c)); returns 1 iff MATCH in nxt. */
static int nfa_step(const orc_regex *r, const uint64_t *src, int c, uint64_t *nxt) {
  memset(nxt, 0, (size_t)r->nw * 8);
  for (int w = 0; w < r->nw; w++) {
    uint64_t bits = src[w];
    while (bits) {
      int q = w * 64 + __builtin_ctzll(bits);
      bits &= bits - 1;
      if (r->st[q].type == S_CHAR && bs_has(&r->st[q].set, c)) {
        const uint64_t *a = r->after + (size_t)q * r->nw;
        for (int k = 0; k < r->nw; k++) nxt[k] |= a[k];
      }
    }
  }
  int m = r->match_state;
  return (int)((nxt[m >> 6] >> (m & 63)) & 1);
}

/* ------------------------------------------------------------------ */
/* result sink                                                         */
/* ------------------------------------------------------------------ */
static uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

typedef struct {
  uint32_t *dense;     /* nullable: LSB-first bitstream, bit p = position p */
  uint64_t *pos;       /* nullable: match-end positions, ascending */
  uint64_t pos_cap;
  uint64_t count, d1, d2;
} sink;

static void emit(sink *k, uint64_t p) {
  if (k->dense) k->dense[p >> 5] |= 1u << (p & 31);
  if (k->pos && k->count < k->pos_cap) k->pos[k->count] = p;
  k->count++;
  k->d1 += splitmix64(p);
  k->d2 += splitmix64(p ^ 0x9E3779B97F4A7C15ull);
}

/* Plain Thompson simulation, SURVEY.md Sec. 8(c) steps 2-3. */
static void run_uncached(const orc_regex *r, const uint8_t *in, uint64_t len, sink *k) {
  uint64_t *cur = (uint64_t *)calloc((size_t)r->nw, 8);
  uint64_t *src = (uint64_t *)calloc((size_t)r->nw, 8);
  uint64_t *nxt = (uint64_t *)calloc((size_t)r->nw, 8);
  for (uint64_t i = 0; i < len; i++) {
    for (int w = 0; w < r->nw; w++) src[w] = cur[w] | r->start[w]; /* inject starts before stepping */
    if (nfa_step(r, src, in[i], nxt)) emit(k, i);
    uint64_t *t = cur; cur = nxt; nxt = t;
  }
  free(cur);
  free(src);
  free(nxt);
}

/* Memoised (lazy DFA) simulation; DFA state = src set (always contains start).
 * trans[d*256+c] = (next_id << 1) | accept, or UINT32_MAX if not computed. */
typedef struct {
  int nw;
  uint64_t *keys; /* nkeys * nw */
  uint32_t *trans;
  int nkeys, cap;
  int32_t *hash; /* open addressing, size hcap */
  int hcap;
} dfa;

static uint64_t key_hash(const uint64_t *k, int nw) {
  uint64_t h = 0x12345678ull;
  for (int i = 0; i < nw; i++) h = splitmix64(h ^ k[i]);
  return h;
}

static void dfa_reset(dfa *d) {
  d->nkeys = 0;
  for (int i = 0; i < d->hcap; i++) d->hash[i] = -1;
}

static int dfa_lookup(dfa *d, const uint64_t *key) {
  uint64_t h = key_hash(key, d->nw) & (uint64_t)(d->hcap - 1);
  for (;;) {
    int id = d->hash[h];
    if (id < 0) break;
    if (!memcmp(d->keys + (size_t)id * d->nw, key, (size_t)d->nw * 8)) return id;
    h = (h + 1) & (uint64_t)(d->hcap - 1);
  }
  if (d->nkeys == d->cap) return -1; /* full */
  int id = d->nkeys++;
  memcpy(d->keys + (size_t)id * d->nw, key, (size_t)d->nw * 8);
  for (int c = 0; c < 256; c++) d->trans[(size_t)id * 256 + c] = UINT32_MAX;
  d->hash[h] = id;
  return id;
}

static void run_cached(const orc_regex *r, const uint8_t *in, uint64_t len, sink *k, int max_states) {
  dfa d;
  memset(&d, 0, sizeof d);
  d.nw = r->nw;
  d.cap = max_states;
  d.hcap = 1;
  while (d.hcap < 2 * max_states) d.hcap <<= 1;
  d.keys = (uint64_t *)malloc((size_t)d.cap * d.nw * 8);
  d.trans = (uint32_t *)malloc((size_t)d.cap * 256 * 4);
  d.hash = (int32_t *)malloc((size_t)d.hcap * 4);
  uint64_t *tmp = (uint64_t *)calloc((size_t)r->nw, 8);
  uint64_t *cur = (uint64_t *)calloc((size_t)r->nw, 8); /* current src set */
  dfa_reset(&d);
  memcpy(cur, r->start, (size_t)r->nw * 8);
  int s = dfa_lookup(&d, cur);
  for (uint64_t i = 0; i < len; i++) {
    int c = in[i];
    uint32_t t = d.trans[(size_t)s * 256 + c];
    if (t == UINT32_MAX) {
      const uint64_t *src = d.keys + (size_t)s * d.nw;
      int acc = nfa_step(r, src, c, tmp);
      for (int w = 0; w < r->nw; w++) tmp[w] |= r->start[w];
      int ns = dfa_lookup(&d, tmp);
      if (ns < 0) { /* cache full: flush, keep only the new state */
        dfa_reset(&d);
        ns = dfa_lookup(&d, tmp);
        t = ((uint32_t)ns << 1) | (uint32_t)acc;
        s = ns;
        if (acc) emit(k, i);
        continue;
      }
      t = ((uint32_t)ns << 1) | (uint32_t)acc;
      d.trans[(size_t)s * 256 + c] = t;
    }
    if (t & 1) emit(k, i);
    s = (int)(t >> 1);
  }
  free(tmp);
  free(cur);
  free(d.keys);
  free(d.trans);
  free(d.hash);
}

/* Single regex.  dense: nullable, ceil(len/32) words, zeroed by the caller.
 * pos: nullable, capacity pos_cap.  Returns the match count. */
uint64_t orc_run(const orc_regex *r, const uint8_t *in, uint64_t len, int use_cache, int max_states,
                 uint32_t *dense, uint64_t *pos, uint64_t pos_cap, uint64_t *d1, uint64_t *d2) {
  sink k;
  memset(&k, 0, sizeof k);
  k.dense = dense;
  k.pos = pos;
  k.pos_cap = pos_cap;
  if (use_cache) run_cached(r, in, len, &k, max_states > 0 ? max_states : 4096);
  else run_uncached(r, in, len, &k);
  if (d1) *d1 = k.d1;
  if (d2) *d2 = k.d2;
  return k.count;
}

/* ------------------------------------------------------------------ */
/* pattern set, thread pool over regexes   */
/* ------------------------------------------------------------------ */
typedef struct {
  orc_regex **rs;
  uint32_t n;
  const uint8_t *in;
  uint64_t len;
  int use_cache, max_states;
  uint32_t *dense;
  uint64_t pitch;
  uint64_t *counts, *digests;
  uint32_t next; /* work queue */
  pthread_mutex_t mu;
} set_job;

static void *set_worker(void *arg) {
  set_job *j = (set_job *)arg;
  for (;;) {
    pthread_mutex_lock(&j->mu);
    uint32_t r = j->next++;
    pthread_mutex_unlock(&j->mu);
    if (r >= j->n) break;
    uint64_t d1 = 0, d2 = 0;
    uint32_t *dn = j->dense ? j->dense + (uint64_t)r * j->pitch : NULL;
    uint64_t c = orc_run(j->rs[r], j->in, j->len, j->use_cache, j->max_states, dn, NULL, 0, &d1, &d2);
    if (j->counts) j->counts[r] = c;
    if (j->digests) {
      j->digests[2 * (uint64_t)r] = d1;
      j->digests[2 * (uint64_t)r + 1] = d2;
    }
  }
  return NULL;
}

/* Returns 0 on success, else the first failing pattern's error code, with
 * *bad = its index. */
int orc_run_set(const char *const *pats, const size_t *lens, uint32_t n, const uint8_t *in, uint64_t len,
                int threads, int use_cache, int max_states, uint32_t *dense, uint64_t pitch_words,
                uint64_t *counts, uint64_t *digests, uint32_t *bad) {
  orc_regex **rs = (orc_regex **)calloc(n ? n : 1, sizeof(orc_regex *));
  for (uint32_t i = 0; i < n; i++) {
    int e = orc_compile(pats[i], lens[i], &rs[i], NULL, NULL, 0);
    if (e) {
      if (bad) *bad = i;
      for (uint32_t k = 0; k < i; k++) orc_free(rs[k]);
      free(rs);
      return e;
    }
  }
  set_job j;
  memset(&j, 0, sizeof j);
  j.rs = rs;
  j.n = n;
  j.in = in;
  j.len = len;
  j.use_cache = use_cache;
  j.max_states = max_states;
  j.dense = dense;
  j.pitch = pitch_words;
  j.counts = counts;
  j.digests = digests;
  pthread_mutex_init(&j.mu, NULL);
  if (threads < 1) threads = 1;
  pthread_t *th = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)threads);
  for (int t = 0; t < threads; t++) pthread_create(&th[t], NULL, set_worker, &j);
  for (int t = 0; t < threads; t++) pthread_join(th[t], NULL);
  free(th);
  pthread_mutex_destroy(&j.mu);
  for (uint32_t i = 0; i < n; i++) orc_free(rs[i]);
  free(rs);
  return 0;
}

uint64_t orc_splitmix64(uint64_t x) { return splitmix64(x); }
