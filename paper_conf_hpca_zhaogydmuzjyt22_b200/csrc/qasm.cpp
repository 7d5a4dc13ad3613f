// a1: OpenQASM-2 subset loader (the paper exports its benchmarks as OpenQASM,
// P:409, format ref [14] P:485). Registers are concatenated in declaration order (first
// register = low qubits); `creg`, `measure`, `barrier` are accepted and ignored (P:81:
// measurement at the end only); `gate`, `opaque`, `reset`, `if` are rejected UNSUPPORTED.
#include <cctype>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <map>
#include <unordered_map>
#include <string>
#include <string_view>
#include <vector>

#include "qgpu_internal.h"

namespace qgpu {
namespace {

enum TokKind { T_EOF, T_ID, T_NUM, T_STR, T_SYM, T_ARROW };

struct Tok {
  TokKind k;
  std::string_view s;  // view into the source text (which outlives the parse)
  double v = 0;
  int line, col;
};

struct ParseError {
  qgpu_status code;
  std::string msg;
};

class Lexer {
 public:
  Lexer(const char* t, size_t n) : p_(t), e_(t + n) {}
  std::vector<Tok> run() {
    std::vector<Tok> out;
    out.reserve(size_t(e_ - p_) / 3 + 16);
    for (;;) {
      skip();
      Tok t{T_EOF, "", 0, line_, col()};
      if (p_ >= e_) { out.push_back(t); return out; }
      const char c = *p_;
      if (std::isalpha((unsigned char)c) || c == '_') {
        const char* s = p_;
        while (p_ < e_ && (std::isalnum((unsigned char)*p_) || *p_ == '_')) ++p_;
        t.k = T_ID; t.s = std::string_view(s, size_t(p_ - s));
      } else if (std::isdigit((unsigned char)c) || (c == '.' && p_ + 1 < e_ && std::isdigit((unsigned char)p_[1]))) {
        const char* s = p_;
        while (p_ < e_ && (std::isdigit((unsigned char)*p_) || *p_ == '.')) ++p_;
        if (p_ < e_ && (*p_ == 'e' || *p_ == 'E')) {
          const char* q = p_ + 1;
          if (q < e_ && (*q == '+' || *q == '-')) ++q;
          if (q < e_ && std::isdigit((unsigned char)*q)) {
            p_ = q;
            while (p_ < e_ && std::isdigit((unsigned char)*p_)) ++p_;
          }
        }
        t.k = T_NUM; t.s = std::string_view(s, size_t(p_ - s));
        // plain integers (qubit indices, most numbers in a circuit) exactly, without strtod
        bool integral = t.s.size() <= 15;
        uint64_t iv = 0;
        for (char ch : t.s) {
          if (ch < '0' || ch > '9') { integral = false; break; }
          iv = iv * 10 + uint64_t(ch - '0');
        }
        t.v = integral ? double(iv) : std::strtod(std::string(t.s).c_str(), nullptr);
      } else if (c == '"') {
        const char* s = ++p_;
        while (p_ < e_ && *p_ != '"' && *p_ != '\n') ++p_;
        if (p_ >= e_ || *p_ != '"') throw ParseError{QGPU_ERR_PARSE, at(t) + "unterminated string"};
        t.k = T_STR; t.s = std::string_view(s, size_t(p_ - s)); ++p_;
      } else if (c == '-' && p_ + 1 < e_ && p_[1] == '>') {
        t.k = T_ARROW; t.s = std::string_view(p_, 2); p_ += 2;
      } else if (c != '\0' && std::strchr(";,[](){}+-*/^", c) != nullptr) {
        t.k = T_SYM; t.s = std::string_view(p_, 1); ++p_;
      } else {
        throw ParseError{QGPU_ERR_PARSE, at(t) + "unexpected character '" + std::string(1, c) + "'"};
      }
      out.push_back(std::move(t));
    }
  }
  static std::string at(const Tok& t) {
    return "line " + std::to_string(t.line) + ":" + std::to_string(t.col) + ": ";
  }

 private:
  void skip() {
    while (p_ < e_) {
      if (*p_ == '\n') { ++line_; ++p_; lstart_ = p_; }
      else if (*p_ == ' ' || *p_ == '\t' || *p_ == '\r') ++p_;
      else if (*p_ == '/' && p_ + 1 < e_ && p_[1] == '/') { while (p_ < e_ && *p_ != '\n') ++p_; }
      else break;
    }
  }
  int col() const { return int(p_ - lstart_) + 1; }
  const char* p_;
  const char* e_;
  const char* lstart_ = p_;
  int line_ = 1;
};

class Parser {
 public:
  explicit Parser(std::vector<Tok> t) : t_(std::move(t)) {}

  void run(Circuit* c) {
    if (peek().k == T_ID && peek().s == "OPENQASM") {
      next();
      if (peek().k != T_NUM) fail(peek(), "expected version");
      next();
      expect(';');
    }
    while (peek().k != T_EOF) {
      const Tok& t = next();
      if (t.k != T_ID) fail(t, "unexpected token '" + std::string(t.s) + "'");
      if (t.s == "include") {
        if (peek().k != T_STR) fail(peek(), "expected file name");
        next();
        expect(';');
      } else if (t.s == "qreg" || t.s == "creg") {
        const Tok& name = next();
        if (name.k != T_ID) fail(name, "expected register name");
        expect('[');
        const Tok& sz = next();
        if (sz.k != T_NUM) fail(sz, "expected register size");
        expect(']');
        expect(';');
        if (t.s == "qreg") {
          if (regs_.count(name.s)) fail(name, "duplicate register", QGPU_ERR_INVALID_ARG);
          regs_[std::string(name.s)] = {n_, int(sz.v)};
          n_ += int(sz.v);
          if (n_ > kMaxQubits) fail(sz, "too many qubits", QGPU_ERR_UNSUPPORTED);
        }
      } else if (t.s == "measure" || t.s == "barrier") {
        while (peek().k != T_EOF && !is(';')) next();
        expect(';');
      } else if (t.s == "gate" || t.s == "opaque" || t.s == "reset" || t.s == "if") {
        fail(t, "'" + std::string(t.s) + "' is not supported", QGPU_ERR_UNSUPPORTED);
      } else {
        gate(t, c);
      }
    }
    c->n = n_;
  }

 private:
  const Tok& peek() const { return t_[i_]; }
  const Tok& next() { return t_[i_ < t_.size() - 1 ? i_++ : i_]; }
  bool is(char ch) const { return peek().k == T_SYM && peek().s[0] == ch; }  // symbols: 1 char
  void expect(char ch) {
    if (!is(ch)) fail(peek(), std::string("expected '") + ch + "', got '" + std::string(peek().s) + "'");
    next();
  }
  [[noreturn]] void fail(const Tok& t, const std::string& m, qgpu_status c = QGPU_ERR_PARSE) {
    throw ParseError{c, Lexer::at(t) + m};
  }

  // expression grammar: expr := term (('+'|'-') term)*; term := unary (('*'|'/') unary)*;
  // unary := ('-'|'+') unary | power; power := primary ('^' unary)?
  double expr() {
    double v = term();
    while (is('+') || is('-')) {
      const bool add = next().s[0] == '+';
      const double r = term();
      v = add ? v + r : v - r;
    }
    return v;
  }
  double term() {
    double v = unary();
    while (is('*') || is('/')) {
      const bool mul = next().s[0] == '*';
      const double r = unary();
      v = mul ? v * r : v / r;
    }
    return v;
  }
  double unary() {
    if (is('-')) { next(); return -unary(); }
    if (is('+')) { next(); return unary(); }
    return power();
  }
  double power() {
    const double b = primary();
    if (is('^')) { next(); return std::pow(b, unary()); }
    return b;
  }
  double primary() {
    const Tok& t = next();
    if (t.k == T_NUM) return t.v;
    if (t.k == T_ID) {
      if (t.s == "pi") return M_PI;
      static const std::map<std::string, double (*)(double), std::less<>> f = {
          {"sin", [](double x) { return std::sin(x); }},  {"cos", [](double x) { return std::cos(x); }},
          {"tan", [](double x) { return std::tan(x); }},  {"exp", [](double x) { return std::exp(x); }},
          {"ln", [](double x) { return std::log(x); }},   {"sqrt", [](double x) { return std::sqrt(x); }}};
      auto it = f.find(t.s);
      if (it == f.end()) fail(t, "unknown identifier '" + std::string(t.s) + "' in expression");
      expect('(');
      const double v = expr();
      expect(')');
      return it->second(v);
    }
    if (t.k == T_SYM && t.s[0] == '(') {
      const double v = expr();
      expect(')');
      return v;
    }
    fail(t, "unexpected token '" + std::string(t.s) + "' in expression");
  }

  std::vector<int> operand() {
    const Tok& t = next();
    const auto rit = t.k == T_ID ? regs_.find(t.s) : regs_.end();
    if (rit == regs_.end()) fail(t, "unknown register '" + std::string(t.s) + "'");
    const auto r = rit->second;
    if (is('[')) {
      next();
      const Tok& i = next();
      if (i.k != T_NUM) fail(i, "expected index");
      expect(']');
      const int idx = int(i.v);
      if (idx < 0 || idx >= r.second) fail(i, "index out of range", QGPU_ERR_INVALID_ARG);
      return {r.first + idx};
    }
    std::vector<int> all;
    for (int k = 0; k < r.second; ++k) all.push_back(r.first + k);
    return all;
  }

  // One gate statement. Its matrix depends only on the gate name and the parameter text (the
  // expressions use constants only), so statements that repeat both -- most of a generated
  // circuit -- reuse the matrix and flags built the first time (memo_, per parse).
  void gate(const Tok& t, Circuit* c) {
    int np, nq, nc;
    cplx U[16];
    // memo key: the name and the raw source text of the parameter list
    size_t close = i_;
    if (is('(')) {
      int depth = 0;
      for (close = i_; t_[close].k != T_EOF; ++close) {
        if (t_[close].k == T_SYM && t_[close].s[0] == '(') ++depth;
        if (t_[close].k == T_SYM && t_[close].s[0] == ')' && --depth == 0) break;
      }
    }
    std::string key(t.s);
    if (close != i_ && t_[close].k != T_EOF)
      key.append(t_[i_].s.data(), size_t(t_[close].s.data() - t_[i_].s.data()) + 1);
    const bool memo_ok = close == i_ || t_[close].k != T_EOF;  // an unclosed list: parse, fail
    auto hit = memo_ok ? memo_.find(key) : memo_.end();
    const Memo* m = nullptr;
    if (hit != memo_.end()) {
      m = &hit->second;
      i_ = close == i_ ? i_ : close + 1;  // the parameter list was evaluated before
      np = m->np; nq = m->nq; nc = m->nc;
    } else {
      const std::string name(t.s);
      if (!gate_matrix(name, {}, &np, &nq, &nc, U, false))
        fail(t, "unknown gate '" + std::string(t.s) + "'", QGPU_ERR_UNSUPPORTED);
      std::vector<double> p;
      if (is('(')) {
        next();
        if (!is(')')) {
          p.push_back(expr());
          while (is(',')) { next(); p.push_back(expr()); }
        }
        expect(')');
      }
      if (int(p.size()) != np)
        fail(t, std::string(t.s) + " takes " + std::to_string(np) + " parameters", QGPU_ERR_INVALID_ARG);
      Memo e;
      e.np = np; e.nq = nq; e.nc = nc;
      gate_matrix(name, p, &np, &nq, &nc, e.U, true);
      const int nt = nq - nc;
      e.diag = is_diagonal(e.U, nt);
      e.swap = is_swap_matrix(e.U, nt);
      m = &memo_.emplace(std::move(key), e).first->second;  // unordered_map: stable addresses
    }
    std::vector<std::vector<int>> ops{operand()};
    while (is(',')) { next(); ops.push_back(operand()); }
    expect(';');
    if (int(ops.size()) != nq)
      fail(t, std::string(t.s) + " takes " + std::to_string(nq) + " qubits", QGPU_ERR_INVALID_ARG);
    size_t width = 1;
    for (auto& o : ops) width = std::max(width, o.size());
    for (auto& o : ops)
      if (o.size() != 1 && o.size() != width) fail(t, "register size mismatch", QGPU_ERR_INVALID_ARG);
    (void)U;
    const int nt = nq - nc;
    for (size_t k = 0; k < width; ++k) {
      Gate g;
      g.nt = nt;
      g.line = t.line;
      uint64_t seen = 0;
      for (int j = 0; j < nq; ++j) {
        const int q = ops[j].size() == 1 ? ops[j][0] : ops[j][k];
        if (seen >> q & 1) fail(t, "repeated qubit operand", QGPU_ERR_INVALID_ARG);
        seen |= 1ull << q;
        if (j < nc) g.cmask |= 1ull << q;
        else g.t[j - nc] = q;
      }
      for (int i = 0; i < (1 << (2 * nt)); ++i) g.U[i] = m->U[i];
      g.diag = m->diag;
      g.relabel = (g.cmask == 0 && m->swap);
      c->gates.push_back(g);
    }
  }

  std::vector<Tok> t_;
  size_t i_ = 0;
  int n_ = 0;
  std::map<std::string, std::pair<int, int>, std::less<>> regs_;
  struct Memo {
    int np, nq, nc;
    bool diag, swap;
    cplx U[16];
  };
  std::unordered_map<std::string, Memo> memo_;
};

}  // namespace

qgpu_status parse_qasm(const char* text, size_t len, Circuit* out, std::string* err) {
  try {
    Lexer lx(text, len);
    Parser ps(lx.run());
    Circuit c;
    c.gates.reserve(len / 12 + 16);  // a gate statement takes >= ~12 source bytes in practice
    ps.run(&c);
    *out = std::move(c);
    return QGPU_OK;
  } catch (const ParseError& e) {
    *err = e.msg;
    return e.code;
  } catch (const std::exception& e) {
    *err = e.what();
    return QGPU_ERR_PARSE;
  }
}

}  // namespace qgpu
