python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
P1='n0 = 1.\nn1 = if (v > sqrt(007 / w)) then (if (10 > norm(grad(n0))) then ((0.5 <= u)) else (u - w)) else (-0.0 / u + u)\n\n# tail comment\n'
P2='n0 = v\nt1 = sqrt(grad(u)[1])\nn2 = if (if (w > 0.0) then (w) else (1) > u) then (0.0) else ((v))\nn3 = 0.0\nt1 = grad(n2*w)[2] / ((v <= u))\n\n# tail comment\n'
for v in ieee exact markstein; do
  echo "P1 $v"; python tools/fuzz_probe.py "$P1" 22 8 9 f64 $v
  echo "P2 $v"; python tools/fuzz_probe.py "$P2" 24 13 9 f32 $v
done
