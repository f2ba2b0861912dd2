// Expression language -> dataflow network.
//
// A hand-written lexer + recursive-descent parser for the VisIt-style
// language of the paper (Fig. 3; intro expression L19) and the
// lowering of the parse tree into the network specification: generic filter
// ids in encounter order (L72), operators -> filter names and v[k] ->
// decompose (L74), constants reduced to single sources and a limited,
// syntactic common-subexpression elimination (L76).  Grammar, precedence,
// constant parsing, error classes and the canonical text are DESIGN.md
// readings R2-R10.
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "common.hpp"

namespace dfg {

enum class Op : int {
  Const, Add, Sub, Mult, Div, Neg, Sqrt,
  Gt, Lt, Ge, Le, Eq, Ne, Select,
  Decompose, Compose, Grad3d
};
const char* op_name(Op op);
int op_arity(Op op);  // number of non-mesh inputs; -1 = variable (compose)

// A reference to a value: a filter result, a bound input field, or one of
// the mesh arrays (dims/x/y/z; only ever an input of grad3d).
struct Ref {
  enum Kind : int { Filter, Input, Mesh } kind = Filter;
  int id = -1;          // filter index, input index, or mesh index (0..3)
  bool operator==(const Ref& o) const { return kind == o.kind && id == o.id; }
};

struct Filter {
  Op op;
  std::vector<Ref> in;  // immediate inputs (L72); grad3d: f, dims, x, y, z
  double cval = 0;      // Const: the literal parsed to T (exact in double)
  int k = -1;           // Decompose: lane
  int width = 1;        // 1 = scalar; n = vector with n used lanes
  bool has_grad = false;
};

struct Dag {
  DType dtype = DType::F32;
  std::vector<std::string> inputs;          // bound input names
  std::vector<Filter> filters;              // network order (emission order)
  std::vector<std::pair<std::string, Ref>> names;
  Ref result;
  int width(const Ref& r) const { return r.kind == Ref::Filter ? filters[r.id].width : 1; }
  std::string ref_text(const Ref& r) const;
  std::string dump() const;                 // canonical text, R10
};

// Throws DfgError with DFG_E_PARSE / DFG_E_UNDEFINED / DFG_E_TYPE.
Dag build_dag(const std::string& src, const std::vector<std::string>& inputs, DType dtype);

bool valid_input_name(const std::string& name);
std::string hexfloat(double v);

}  // namespace dfg
