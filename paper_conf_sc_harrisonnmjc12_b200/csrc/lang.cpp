// Expression language -> dataflow network.  See lang.hpp for the paper
// passages; R2-R10 for the readings this code implements.
#include "lang.hpp"

#include <clocale>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <locale.h>
#include <map>
#include <memory>
#include <sstream>

namespace dfg {

namespace {

const char* kMeshNames[4] = {"dims", "x", "y", "z"};

int mesh_index(const std::string& s) {
  for (int i = 0; i < 4; ++i)
    if (s == kMeshNames[i]) return i;
  return -1;
}

bool is_keyword(const std::string& s) { return s == "if" || s == "then" || s == "else"; }

bool is_fref(const std::string& s) {
  if (s.size() < 2 || s[0] != 'f') return false;
  for (size_t i = 1; i < s.size(); ++i)
    if (s[i] < '0' || s[i] > '9') return false;
  return true;
}

bool is_alpha_(char c) { return (c >= 'A' && c <= 'Z') || (c >= 'a' && c <= 'z') || c == '_'; }
bool is_digit(char c) { return c >= '0' && c <= '9'; }

// ------------------------------------------------------------------ lexer
enum class TK { Number, Int, Ident, Kw, OpTok, Newline, End };

struct Token {
  TK kind;
  std::string text;
  int line, col;
};

bool is_binary_op(const std::string& t) {
  static const char* ops[] = {"+", "-", "*", "/", ">", "<", ">=", "<=", "==", "!="};
  for (auto o : ops)
    if (t == o) return true;
  return false;
}

[[noreturn]] void parse_error(int line, int col, const std::string& what) {
  fail(DFG_E_PARSE, std::to_string(line) + ":" + std::to_string(col) + ": " + what);
}

std::vector<Token> lex(const std::string& s) {
  std::vector<Token> out;
  int depth = 0, line = 1, col = 1;
  size_t i = 0, n = s.size();
  auto push = [&](TK k, std::string t, int l, int c) { out.push_back(Token{k, std::move(t), l, c}); };
  while (i < n) {
    char ch = s[i];
    if (ch == ' ' || ch == '\t' || ch == '\r') { ++i; ++col; continue; }
    if (ch == '#') {
      while (i < n && s[i] != '\n') ++i;
      continue;
    }
    if (ch == '\n') {
      bool keep = depth == 0 && !out.empty() && out.back().kind != TK::Newline;
      if (keep && out.back().kind == TK::OpTok) {
        const std::string& t = out.back().text;
        if (is_binary_op(t) || t == "," || t == "=") keep = false;
      }
      if (keep) push(TK::Newline, "\n", line, col);
      ++i; ++line; col = 1;
      continue;
    }
    bool starts_number = is_digit(ch) || (ch == '.' && i + 1 < n && is_digit(s[i + 1]));
    if (starts_number) {
      size_t j = i;
      bool integral = true;
      if (is_digit(s[j])) {
        while (j < n && is_digit(s[j])) ++j;
        if (j < n && s[j] == '.') {
          integral = false;
          ++j;
          while (j < n && is_digit(s[j])) ++j;
        }
      } else {  // '.' digits+
        integral = false;
        ++j;
        while (j < n && is_digit(s[j])) ++j;
      }
      if (j < n && (s[j] == 'e' || s[j] == 'E')) {
        size_t e = j + 1;
        if (e < n && (s[e] == '+' || s[e] == '-')) ++e;
        if (e < n && is_digit(s[e])) {
          while (e < n && is_digit(s[e])) ++e;
          j = e;
          integral = false;
        }
      }
      push(integral ? TK::Int : TK::Number, s.substr(i, j - i), line, col);
      col += int(j - i);
      i = j;
      continue;
    }
    if (is_alpha_(ch)) {
      size_t j = i;
      while (j < n && (is_alpha_(s[j]) || is_digit(s[j]))) ++j;
      std::string t = s.substr(i, j - i);
      push(is_keyword(t) ? TK::Kw : TK::Ident, t, line, col);
      col += int(j - i);
      i = j;
      continue;
    }
    if (i + 1 < n) {
      std::string two = s.substr(i, 2);
      if (two == ">=" || two == "<=" || two == "==" || two == "!=") {
        push(TK::OpTok, two, line, col);
        i += 2; col += 2;
        continue;
      }
    }
    if (std::strchr("=+-*/()[]{},<>", ch) && ch != '\0') {
      if (ch == '(' || ch == '[' || ch == '{') ++depth;
      else if (ch == ')' || ch == ']' || ch == '}') depth = depth > 0 ? depth - 1 : 0;
      push(TK::OpTok, std::string(1, ch), line, col);
      ++i; ++col;
      continue;
    }
    parse_error(line, col, std::string("unexpected character '") + ch + "'");
  }
  push(TK::End, "", line, col);
  return out;
}

// ------------------------------------------------------------- parse tree
struct Node {
  enum Kind { Num, Ident, Call, Index, Neg, Bin, If, Compose } kind;
  std::string text;                       // Num literal, Ident/Call name, Bin operator
  long long k = 0;                        // Index lane (saturated)
  std::vector<std::unique_ptr<Node>> kids;
};
using NodeP = std::unique_ptr<Node>;

NodeP mk(Node::Kind k, std::string t = "") {
  NodeP n(new Node);
  n->kind = k;
  n->text = std::move(t);
  return n;
}

struct Stmt {
  std::string name;
  NodeP expr;
};

class Parser {
 public:
  explicit Parser(std::vector<Token> t) : t_(std::move(t)) {}

  std::vector<Stmt> program() {
    std::vector<Stmt> stmts;
    while (peek().kind == TK::Newline) next();
    if (peek().kind == TK::End) err(peek(), "empty program");
    for (;;) {
      stmts.push_back(stmt());
      if (peek().kind == TK::End) break;
      if (peek().kind != TK::Newline) err(peek(), "expected end of statement");
      while (peek().kind == TK::Newline) next();
      if (peek().kind == TK::End) break;
    }
    return stmts;
  }

 private:
  std::vector<Token> t_;
  size_t p_ = 0;

  const Token& peek() const { return t_[p_]; }
  const Token& next() { return t_[p_++]; }
  bool at_op(const char* s) const { return peek().kind == TK::OpTok && peek().text == s; }

  [[noreturn]] void err(const Token& tok, const std::string& what) {
    parse_error(tok.line, tok.col, what + " (got '" + (tok.text.empty() ? "<end>" : tok.text) + "')");
  }
  void expect(const char* s) {
    const Token& tok = next();
    if (!((tok.kind == TK::OpTok || tok.kind == TK::Kw) && tok.text == s))
      err(tok, std::string("expected '") + s + "'");
  }

  Stmt stmt() {
    const Token& tok = next();
    if (tok.kind != TK::Ident) err(tok, "expected assignment target");
    if (mesh_index(tok.text) >= 0) err(tok, "cannot assign to reserved name '" + tok.text + "'");
    Stmt st;
    st.name = tok.text;
    expect("=");
    st.expr = expr();
    return st;
  }

  NodeP expr() {
    NodeP a = sum();
    if (peek().kind == TK::OpTok) {
      const std::string& t = peek().text;
      if (t == ">" || t == "<" || t == ">=" || t == "<=" || t == "==" || t == "!=") {
        std::string op = next().text;
        NodeP b = sum();
        NodeP n = mk(Node::Bin, op);
        n->kids.push_back(std::move(a));
        n->kids.push_back(std::move(b));
        return n;
      }
    }
    return a;
  }

  NodeP sum() {
    NodeP a = prod();
    while (at_op("+") || at_op("-")) {
      std::string op = next().text;
      NodeP n = mk(Node::Bin, op);
      n->kids.push_back(std::move(a));
      n->kids.push_back(prod());
      a = std::move(n);
    }
    return a;
  }

  NodeP prod() {
    NodeP a = unary();
    while (at_op("*") || at_op("/")) {
      std::string op = next().text;
      NodeP n = mk(Node::Bin, op);
      n->kids.push_back(std::move(a));
      n->kids.push_back(unary());
      a = std::move(n);
    }
    return a;
  }

  NodeP unary() {
    if (at_op("-")) {
      next();
      NodeP n = mk(Node::Neg);
      n->kids.push_back(unary());
      return n;
    }
    return postfix();
  }

  NodeP postfix() {
    NodeP a = primary();
    while (at_op("[")) {
      next();
      const Token& tok = next();
      if (tok.kind != TK::Int) err(tok, "expected integer index");
      long long k = 0;
      for (char c : tok.text) {
        k = k * 10 + (c - '0');
        if (k > 1000000) k = 1000000;  // saturate: any such index is out of range
      }
      expect("]");
      NodeP n = mk(Node::Index);
      n->k = k;
      n->kids.push_back(std::move(a));
      a = std::move(n);
    }
    return a;
  }

  NodeP primary() {
    const Token& tok = next();
    if (tok.kind == TK::Number || tok.kind == TK::Int) return mk(Node::Num, tok.text);
    if (tok.kind == TK::Ident) {
      if (at_op("(")) {
        next();
        NodeP n = mk(Node::Call, tok.text);
        if (!at_op(")")) {
          n->kids.push_back(expr());
          while (at_op(",")) {
            next();
            n->kids.push_back(expr());
          }
        }
        expect(")");
        return n;
      }
      return mk(Node::Ident, tok.text);
    }
    if (tok.kind == TK::OpTok && tok.text == "(") {
      NodeP e = expr();
      expect(")");
      return e;
    }
    if (tok.kind == TK::Kw && tok.text == "if") {  // L19
      NodeP n = mk(Node::If);
      expect("(");
      n->kids.push_back(expr());
      expect(")");
      expect("then");
      expect("(");
      n->kids.push_back(expr());
      expect(")");
      expect("else");
      expect("(");
      n->kids.push_back(expr());
      expect(")");
      return n;
    }
    if (tok.kind == TK::OpTok && tok.text == "{") {
      NodeP n = mk(Node::Compose);
      n->kids.push_back(expr());
      expect(",");
      n->kids.push_back(expr());
      while (at_op(",")) {
        next();
        n->kids.push_back(expr());
      }
      expect("}");
      return n;
    }
    err(tok, "expected expression");
  }
};

// ---------------------------------------------------------------- lowering
locale_t c_locale() {
  static locale_t loc = newlocale(LC_ALL_MASK, "C", (locale_t)0);
  return loc;
}

double parse_const(const std::string& text, DType dt) {
  // Direct decimal -> T rounding (strtof for float: no double rounding), R5.
  if (dt == DType::F32) return double(strtof_l(text.c_str(), nullptr, c_locale()));
  return strtod_l(text.c_str(), nullptr, c_locale());
}

class Lowerer {
 public:
  Lowerer(DType dt, const std::vector<std::string>& inputs) {
    dag_.dtype = dt;
    dag_.inputs = inputs;
  }

  Dag run(std::vector<Stmt>& stmts) {
    Ref ref;
    for (auto& st : stmts) {
      ref = lower(*st.expr);  // RHS before the LHS is (re)bound
      env_[st.name] = ref;
      dag_.names.emplace_back(st.name, ref);
    }
    dag_.result = ref;
    return std::move(dag_);
  }

 private:
  Dag dag_;
  std::map<std::string, Ref> env_;
  std::map<std::string, int> cse_;

  Ref emit(Op op, std::vector<Ref> in, double cval, int k, int width) {
    std::ostringstream key;
    key << int(op) << '|';
    if (op == Op::Const) {
      if (dag_.dtype == DType::F32) {
        float f = float(cval);
        uint32_t b;
        std::memcpy(&b, &f, 4);
        key << b;
      } else {
        uint64_t b;
        std::memcpy(&b, &cval, 8);
        key << b;
      }
    } else {
      for (auto& r : in) key << int(r.kind) << ':' << r.id << ',';
      key << '|' << k;
    }
    auto it = cse_.find(key.str());
    if (it != cse_.end()) return Ref{Ref::Filter, it->second};  // L76
    Filter f;
    f.op = op;
    f.in = std::move(in);
    f.cval = cval;
    f.k = k;
    f.width = width;
    f.has_grad = op == Op::Grad3d;
    for (auto& r : f.in)
      if (r.kind == Ref::Filter && dag_.filters[r.id].has_grad) f.has_grad = true;
    dag_.filters.push_back(std::move(f));
    int id = int(dag_.filters.size()) - 1;
    cse_[key.str()] = id;
    return Ref{Ref::Filter, id};
  }

  void need_scalar(const Ref& r, const std::string& what) {
    if (dag_.width(r) != 1) fail(DFG_E_TYPE, what + ": expected a scalar operand");
  }

  Ref lower(Node& n) {
    switch (n.kind) {
      case Node::Num:
        return emit(Op::Const, {}, parse_const(n.text, dag_.dtype), -1, 1);
      case Node::Ident: {
        auto it = env_.find(n.text);
        if (it != env_.end()) return it->second;
        for (size_t i = 0; i < dag_.inputs.size(); ++i)
          if (dag_.inputs[i] == n.text) return Ref{Ref::Input, int(i)};
        if (mesh_index(n.text) >= 0) fail(DFG_E_TYPE, "mesh array '" + n.text + "' used as a field");
        fail(DFG_E_UNDEFINED, "unknown identifier '" + n.text + "'");
      }
      case Node::Call:
        return call(n);
      case Node::Index: {
        Ref b = lower(*n.kids[0]);
        int w = dag_.width(b);
        if (w == 1) fail(DFG_E_TYPE, "decompose of a scalar");
        if (n.k >= w) fail(DFG_E_TYPE, "decompose index " + std::to_string(n.k) + " out of range");
        return emit(Op::Decompose, {b}, 0, int(n.k), 1);
      }
      case Node::Neg: {
        Ref x = lower(*n.kids[0]);
        need_scalar(x, "unary -");
        return emit(Op::Neg, {x}, 0, -1, 1);
      }
      case Node::Bin: {
        Ref a = lower(*n.kids[0]);
        Ref b = lower(*n.kids[1]);
        need_scalar(a, n.text);
        need_scalar(b, n.text);
        static const std::map<std::string, Op> ops = {
            {"+", Op::Add}, {"-", Op::Sub}, {"*", Op::Mult}, {"/", Op::Div},
            {">", Op::Gt},  {"<", Op::Lt},  {">=", Op::Ge},  {"<=", Op::Le},
            {"==", Op::Eq}, {"!=", Op::Ne}};
        return emit(ops.at(n.text), {a, b}, 0, -1, 1);
      }
      case Node::If: {
        Ref c = lower(*n.kids[0]);
        Ref t = lower(*n.kids[1]);
        Ref e = lower(*n.kids[2]);
        need_scalar(c, "if");
        need_scalar(t, "if");
        need_scalar(e, "if");
        return emit(Op::Select, {c, t, e}, 0, -1, 1);
      }
      case Node::Compose: {
        if (n.kids.size() > 4) fail(DFG_E_TYPE, "compose of more than 4 components");
        std::vector<Ref> refs;
        for (auto& kid : n.kids) refs.push_back(lower(*kid));
        for (auto& r : refs) need_scalar(r, "compose");
        int w = int(refs.size());
        return emit(Op::Compose, std::move(refs), 0, -1, w);
      }
    }
    fail(DFG_E_INVALID, "internal: bad node");
  }

  Ref call(Node& n) {
    const std::string& f = n.text;
    int arity;
    if (f == "sqrt" || f == "grad" || f == "norm") arity = 1;
    else if (f == "grad3d") arity = 5;
    else fail(DFG_E_UNDEFINED, "unknown function '" + f + "'");
    if (int(n.kids.size()) != arity) fail(DFG_E_TYPE, f + " takes " + std::to_string(arity) + " argument(s)");
    if (f == "grad3d") {
      for (int a = 1; a < 5; ++a) {
        const Node& m = *n.kids[a];
        if (!(m.kind == Node::Ident && m.text == kMeshNames[a - 1]))
          fail(DFG_E_TYPE, std::string("grad3d argument ") + std::to_string(a + 1) + " must be '" + kMeshNames[a - 1] + "'");
      }
    }
    Ref x = lower(*n.kids[0]);
    if (f == "sqrt") {
      need_scalar(x, "sqrt");
      return emit(Op::Sqrt, {x}, 0, -1, 1);
    }
    if (f == "grad3d" || f == "grad") {  // grad(f) == grad3d(f, dims, x, y, z)
      need_scalar(x, "grad3d");
      if (x.kind == Ref::Filter && dag_.filters[x.id].has_grad)
        fail(DFG_E_TYPE, "nested grad3d is not supported (halo width 1)");
      std::vector<Ref> in = {x};
      for (int m = 0; m < 4; ++m) in.push_back(Ref{Ref::Mesh, m});
      return emit(Op::Grad3d, std::move(in), 0, -1, 3);
    }
    // norm(v) == sqrt(v[0]*v[0] + v[1]*v[1] + ...), left-associative
    int w = dag_.width(x);
    if (w == 1) fail(DFG_E_TYPE, "norm of a scalar");
    Ref acc;
    for (int k = 0; k < w; ++k) {
      Ref d1 = emit(Op::Decompose, {x}, 0, k, 1);
      Ref d2 = emit(Op::Decompose, {x}, 0, k, 1);
      Ref m = emit(Op::Mult, {d1, d2}, 0, -1, 1);
      acc = k == 0 ? m : emit(Op::Add, {acc, m}, 0, -1, 1);
    }
    return emit(Op::Sqrt, {acc}, 0, -1, 1);
  }
};

}  // namespace

const char* op_name(Op op) {
  switch (op) {
    case Op::Const: return "const";
    case Op::Add: return "add";
    case Op::Sub: return "sub";
    case Op::Mult: return "mult";
    case Op::Div: return "div";
    case Op::Neg: return "neg";
    case Op::Sqrt: return "sqrt";
    case Op::Gt: return "gt";
    case Op::Lt: return "lt";
    case Op::Ge: return "ge";
    case Op::Le: return "le";
    case Op::Eq: return "eq";
    case Op::Ne: return "ne";
    case Op::Select: return "select";
    case Op::Decompose: return "decompose";
    case Op::Compose: return "compose";
    case Op::Grad3d: return "grad3d";
  }
  return "?";
}

int op_arity(Op op) {
  switch (op) {
    case Op::Const: return 0;
    case Op::Neg: case Op::Sqrt: case Op::Decompose: case Op::Grad3d: return 1;
    case Op::Select: return 3;
    case Op::Compose: return -1;
    default: return 2;
  }
}

bool valid_input_name(const std::string& s) {
  if (s.empty() || !is_alpha_(s[0])) return false;
  for (char c : s)
    if (!(is_alpha_(c) || is_digit(c))) return false;
  return !is_keyword(s) && mesh_index(s) < 0 && !is_fref(s);
}

std::string hexfloat(double v) {
  // C99 %a with minimal digits, independent of the locale.
  if (std::isinf(v)) return v > 0 ? "inf" : "-inf";
  if (std::isnan(v)) return "nan";
  uint64_t b;
  std::memcpy(&b, &v, 8);
  bool neg = b >> 63;
  int e = int((b >> 52) & 0x7ff);
  uint64_t m = b & ((uint64_t(1) << 52) - 1);
  std::string s = neg ? "-" : "";
  if (e == 0 && m == 0) return s + "0x0p+0";
  int lead = e == 0 ? 0 : 1;
  int exp = e == 0 ? -1022 : e - 1023;
  static const char* hx = "0123456789abcdef";
  std::string frac;
  for (int i = 12; i >= 0; --i) frac.push_back(hx[(m >> (4 * i)) & 0xf]);
  while (!frac.empty() && frac.back() == '0') frac.pop_back();
  s += "0x";
  s += char('0' + lead);
  if (!frac.empty()) s += "." + frac;
  s += "p";
  s += exp >= 0 ? "+" : "-";
  s += std::to_string(exp >= 0 ? exp : -exp);
  return s;
}

std::string Dag::ref_text(const Ref& r) const {
  switch (r.kind) {
    case Ref::Filter: return "f" + std::to_string(r.id);
    case Ref::Input: return inputs[r.id];
    case Ref::Mesh: return kMeshNames[r.id];
  }
  return "?";
}

std::string Dag::dump() const {
  std::string s = std::string("dfg-dag v1 dtype=") + (dtype == DType::F32 ? "f32" : "f64") + "\n";
  for (size_t k = 0; k < filters.size(); ++k) {
    const Filter& f = filters[k];
    s += "f" + std::to_string(k) + " " + op_name(f.op);
    if (!f.in.empty()) {
      s += " ";
      for (size_t i = 0; i < f.in.size(); ++i) {
        if (i) s += ",";
        s += ref_text(f.in[i]);
      }
    }
    if (f.op == Op::Const) s += " " + hexfloat(f.cval);
    if (f.op == Op::Decompose) s += " " + std::to_string(f.k);
    s += "\n";
  }
  for (auto& nm : names) s += "name " + nm.first + "=" + ref_text(nm.second) + "\n";
  s += "result " + ref_text(result) + "\n";
  return s;
}

Dag build_dag(const std::string& src, const std::vector<std::string>& inputs, DType dtype) {
  for (auto& nm : inputs)
    if (!valid_input_name(nm)) fail(DFG_E_INVALID, "invalid input name '" + nm + "'");
  Parser p(lex(src));
  std::vector<Stmt> stmts = p.program();  // whole program parsed before lowering
  Lowerer lw(dtype, inputs);
  return lw.run(stmts);
}

}  // namespace dfg
