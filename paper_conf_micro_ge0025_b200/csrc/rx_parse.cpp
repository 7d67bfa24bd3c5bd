// rx_parse.cpp -- the compiler's regex front end (grammar of PAPER.md
// character classes, concatenation, alternation, Kleene star,
// R{n,m}, R+, R?; readings c4-c7 of DESIGN.md for '.', escapes, R{n,m}).
//
// Precedence-climbing parser over a token stream.  Independent of the
// oracle's recursive-descent parser (oracle/oracle.c).
#include <cctype>

#include "rx_internal.h"

namespace rx {
namespace {

enum class Tk { End, Char, Set, Dot, LParen, NcLParen, RParen, Bar, Star, Plus, Quest, Brace };

struct Token {
  Tk t = Tk::End;
  int ch = 0;
  ByteSet set;
  int lo = 0, hi = 0;  // Brace
  size_t at = 0;
};

struct Lexer {
  const std::string &s;
  size_t i = 0;
  ParseError *err;
  explicit Lexer(const std::string &src, ParseError *e) : s(src), err(e) {}

  bool bad(int code, size_t at, const char *m) {
    if (err->code == 0) { err->code = code; err->at = at; err->msg = m; }
    return false;
  }

  static int hex(int c) {
    if (c >= '0' && c <= '9') return c - '0';
    c |= 0x20;
    if (c >= 'a' && c <= 'f') return c - 'a' + 10;
    return -1;
  }

  // After a backslash at s[i-1]: one byte (returns 1, *c) or a class (returns 2, *set).
  int escape(int *c, ByteSet *set) {
    size_t at = i - 1;
    if (i >= s.size()) return bad(1, at, "dangling backslash"), 0;
    unsigned char e = (unsigned char)s[i++];
    ByteSet t;
    switch (e) {
      case 'n': *c = 10; return 1;
      case 'r': *c = 13; return 1;
      case 't': *c = 9; return 1;
      case 'f': *c = 12; return 1;
      case 'v': *c = 11; return 1;
      case 'a': *c = 7; return 1;
      case 'x': {
        if (i + 1 >= s.size() + 0 || i + 2 > s.size()) return bad(1, at, "short \\x escape"), 0;
        int h = hex((unsigned char)s[i]), l = hex((unsigned char)s[i + 1]);
        if (h < 0 || l < 0) return bad(1, at, "bad \\x escape"), 0;
        i += 2;
        *c = h * 16 + l;
        return 1;
      }
      case 'd': case 'D': t.range('0', '9'); break;
      case 'w': case 'W': t.range('0', '9'); t.range('a', 'z'); t.range('A', 'Z'); t.set('_'); break;
      case 's': case 'S': for (int x : {9, 10, 11, 12, 13, 32}) t.set(x); break;
      case 'b': case 'B': case 'A': case 'Z': case 'z': case 'G':
        return bad(2, at, "anchor / word-boundary escapes are unsupported"), 0;
      default:
        if (isdigit(e)) return bad(2, at, "backreferences are unsupported"), 0;
        if (isalpha(e)) return bad(1, at, "unknown escape"), 0;
        *c = e;
        return 1;
    }
    if (e == 'D' || e == 'W' || e == 'S') t.invert();
    *set = t;
    return 2;
  }

  bool read_int(int *v) {
    size_t st = i;
    long x = 0;
    while (i < s.size() && isdigit((unsigned char)s[i])) {
      x = x * 10 + (s[i] - '0');
      if (x > 1000000) x = 1000000;
      ++i;
    }
    *v = (int)x;
    return i > st;
  }

  bool next(Token &tk) {
    tk = Token();
    tk.at = i;
    if (i >= s.size()) { tk.t = Tk::End; return true; }
    unsigned char c = (unsigned char)s[i++];
    switch (c) {
      case '(':
        if (i < s.size() && s[i] == '?') {
          if (i + 1 < s.size() && s[i + 1] == ':') { i += 2; tk.t = Tk::NcLParen; return true; }
          return bad(2, tk.at, "group extensions other than (?: are unsupported");
        }
        tk.t = Tk::LParen;
        return true;
      case ')': tk.t = Tk::RParen; return true;
      case '|': tk.t = Tk::Bar; return true;
      case '*': tk.t = Tk::Star; return true;
      case '+': tk.t = Tk::Plus; return true;
      case '?': tk.t = Tk::Quest; return true;
      case '.': tk.t = Tk::Dot; return true;
      case '^': case '$': return bad(2, tk.at, "anchors are unsupported");
      case '{': {
        int a = 0, b = -1;
        bool ha = read_int(&a);
        if (i < s.size() && s[i] == '}') {
          if (!ha) return bad(1, tk.at, "bad {} quantifier");
          ++i;
          b = a;
        } else if (i < s.size() && s[i] == ',') {
          ++i;
          int t = 0;
          bool hb = read_int(&t);
          if (i >= s.size() || s[i] != '}') return bad(1, tk.at, "bad {} quantifier");
          ++i;
          if (!ha) a = 0;
          b = hb ? t : -1;
        } else {
          return bad(1, tk.at, "bad {} quantifier");
        }
        if (b >= 0 && b < a) return bad(1, tk.at, "min repeat greater than max repeat");
        if (a > 1000 || b > 1000) return bad(3, tk.at, "repetition count too large");
        tk.t = Tk::Brace;
        tk.lo = a;
        tk.hi = b;
        return true;
      }
      case '[': return read_class(tk);
      case '\\': {
        int ch = 0;
        ByteSet st;
        int r = escape(&ch, &st);
        if (!r) return false;
        if (r == 1) { tk.t = Tk::Char; tk.ch = ch; }
        else { tk.t = Tk::Set; tk.set = st; }
        return true;
      }
      default:
        tk.t = Tk::Char;
        tk.ch = c;
        return true;
    }
  }

  bool read_class(Token &tk) {
    size_t at = i - 1;
    ByteSet set;
    bool neg = false;
    if (i < s.size() && s[i] == '^') { neg = true; ++i; }
    bool first = true;
    for (;;) {
      if (i >= s.size()) return bad(1, at, "unterminated character class");
      unsigned char c = (unsigned char)s[i];
      if (c == ']' && !first) { ++i; break; }
      first = false;
      int lo;
      ++i;
      if (c == '\\') {
        ByteSet es;
        int r = escape(&lo, &es);
        if (!r) return false;
        if (r == 2) { set.merge(es); continue; }
      } else {
        lo = c;
      }
      if (i + 1 < s.size() && s[i] == '-' && s[i + 1] != ']') {
        ++i;
        int hi;
        unsigned char d = (unsigned char)s[i++];
        if (d == '\\') {
          ByteSet es;
          int r = escape(&hi, &es);
          if (!r) return false;
          if (r == 2) return bad(1, at, "bad character range");
        } else {
          hi = d;
        }
        if (hi < lo) return bad(1, at, "bad character range");
        set.range(lo, hi);
      } else {
        set.set(lo);
      }
    }
    if (neg) set.invert();
    tk.t = Tk::Set;
    tk.set = set;
    return true;
  }
};

struct Parser {
  Lexer lx;
  Token cur;
  ParseError *err;
  int depth = 0;
  Parser(const std::string &s, ParseError *e) : lx(s, e), err(e) {}

  bool advance() { return lx.next(cur); }

  AstP leaf(const ByteSet &s) {
    auto a = std::make_unique<Ast>();
    a->kind = AK::Set;
    a->set = s;
    return a;
  }

  // alt := cat ('|' cat)*
  AstP alt() {
    std::vector<AstP> br;
    br.push_back(cat());
    if (err->code) return nullptr;
    while (cur.t == Tk::Bar) {
      if (!advance()) return nullptr;
      br.push_back(cat());
      if (err->code) return nullptr;
    }
    if (br.size() == 1) return std::move(br[0]);
    auto a = std::make_unique<Ast>();
    a->kind = AK::Alt;
    a->kids = std::move(br);
    return a;
  }

  AstP cat() {
    std::vector<AstP> items;
    while (cur.t != Tk::End && cur.t != Tk::Bar && cur.t != Tk::RParen) {
      AstP p = piece();
      if (err->code) return nullptr;
      items.push_back(std::move(p));
    }
    if (items.empty()) return std::make_unique<Ast>();  // Empty
    if (items.size() == 1) return std::move(items[0]);
    auto a = std::make_unique<Ast>();
    a->kind = AK::Cat;
    a->kids = std::move(items);
    return a;
  }

  AstP piece() {
    AstP at = atom();
    if (err->code) return nullptr;
    bool quantified = false;
    for (;;) {
      int lo, hi;
      if (cur.t == Tk::Star) { lo = 0; hi = -1; }
      else if (cur.t == Tk::Plus) { lo = 1; hi = -1; }
      else if (cur.t == Tk::Quest) { lo = 0; hi = 1; }
      else if (cur.t == Tk::Brace) { lo = cur.lo; hi = cur.hi; }
      else break;
      if (quantified) {
        int code = (cur.t == Tk::Quest || cur.t == Tk::Plus) ? 2 : 1;
        err->code = code;
        err->at = cur.at;
        err->msg = code == 2 ? "lazy / possessive quantifiers are unsupported" : "multiple repeat";
        return nullptr;
      }
      quantified = true;
      auto r = std::make_unique<Ast>();
      r->kind = AK::Rep;
      r->lo = lo;
      r->hi = hi;
      r->kids.push_back(std::move(at));
      at = std::move(r);
      if (!advance()) return nullptr;
    }
    return at;
  }

  AstP atom() {
    Token t = cur;
    switch (t.t) {
      case Tk::Char: {
        ByteSet s;
        s.set(t.ch);
        if (!advance()) return nullptr;
        return leaf(s);
      }
      case Tk::Set: {
        if (!advance()) return nullptr;
        return leaf(t.set);
      }
      case Tk::Dot: {
        ByteSet s;
        s.range(0, 255);
        s.w[0] &= ~(1ull << 10);  // '.' excludes '\n' (reading c4)
        if (!advance()) return nullptr;
        return leaf(s);
      }
      case Tk::LParen:
      case Tk::NcLParen: {
        if (++depth > 200) { err->code = 3; err->at = t.at; err->msg = "nesting too deep"; return nullptr; }
        if (!advance()) return nullptr;
        AstP in = alt();
        if (err->code) return nullptr;
        if (cur.t != Tk::RParen) { err->code = 1; err->at = cur.at; err->msg = "missing )"; return nullptr; }
        --depth;
        if (!advance()) return nullptr;
        return in;
      }
      case Tk::Star: case Tk::Plus: case Tk::Quest: case Tk::Brace:
        err->code = 1; err->at = t.at; err->msg = "nothing to repeat"; return nullptr;
      case Tk::RParen:
        err->code = 1; err->at = t.at; err->msg = "unbalanced )"; return nullptr;
      default:
        err->code = 1; err->at = t.at; err->msg = "unexpected token"; return nullptr;
    }
  }
};

size_t expanded(const Ast &a) {
  switch (a.kind) {
    case AK::Empty: return 0;
    case AK::Set: return 1;
    case AK::Cat: case AK::Alt: {
      size_t n = 0;
      for (auto &k : a.kids) n += expanded(*k);
      return n;
    }
    case AK::Rep: {
      size_t n = expanded(*a.kids[0]);
      size_t copies = a.hi < 0 ? (size_t)(a.lo > 0 ? a.lo : 1) : (size_t)a.hi;
      if (copies == 0) copies = 0;
      return n * (copies ? copies : 0);
    }
  }
  return 0;
}

}  // namespace

AstP parse_regex(const std::string &pat, ParseError &err) {
  err = ParseError{0, 0, ""};
  Parser ps(pat, &err);
  if (!ps.advance()) return nullptr;
  AstP a = ps.alt();
  if (err.code) return nullptr;
  if (ps.cur.t != Tk::End) {
    err.code = 1;
    err.at = ps.cur.at;
    err.msg = "unbalanced )";
    return nullptr;
  }
  return a;
}

bool ast_nullable(const Ast &a) {
  switch (a.kind) {
    case AK::Empty: return true;
    case AK::Set: return false;
    case AK::Cat:
      for (auto &k : a.kids) if (!ast_nullable(*k)) return false;
      return true;
    case AK::Alt:
      for (auto &k : a.kids) if (ast_nullable(*k)) return true;
      return false;
    case AK::Rep: return a.lo == 0 || ast_nullable(*a.kids[0]);
  }
  return false;
}

size_t ast_expanded_size(const Ast &a) { return expanded(a); }

}  // namespace rx
