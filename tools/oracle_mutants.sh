#!/bin/bash
# Mutation check of the oracle's opcode pins (tests/test_oracle_opcodes.py):
# each plausible slip in oracle/kf_oracle.c must make at least one pin fail.
# Restores the source afterwards.  CPU only.  Usage: tools/oracle_mutants.sh
set -u
cd "$(dirname "$0")/.."
cp oracle/kf_oracle.c /tmp/kf_oracle.c.orig
trap 'cp /tmp/kf_oracle.c.orig oracle/kf_oracle.c; rm -f oracle/liboracle.so' EXIT
muts=(
's/pow(a, b)/pow(b, a)/'
's/st\[sp++\] = a < b ? b : (a > c ? c : a); break;/st[sp++] = a < c ? c : (a > b ? b : a); break;/'
's/st\[sp++\] = a > b ? c : d; break; }/st[sp++] = a > b ? d : c; break; }/'
's/b == 0 ? 0 : a \/ b/b == 0 ? 0 : (a - ((a % b + b) % b)) \/ b/'
's/if (a >= o->lut_len) a = o->lut_len - 1;/if (a >= o->lut_len) a = a % o->lut_len;/'
's/case OR_SAT_U8: a = st\[--sp\]; st\[sp++\] = a < 0 ? 0 : (a > 255 ? 255 : a); break;/case OR_SAT_U8: break;/'
's/case OR_SUB: b = st\[--sp\]; a = st\[--sp\]; st\[sp++\] = chk(a - b)/case OR_SUB: a = st[--sp]; b = st[--sp]; st[sp++] = chk(a - b)/'
's/return v >= 0 ? v \/ d : -((-v + d - 1) \/ d);/return v \/ d;/'
's/case OR_DIV: b = st\[--sp\]; a = st\[--sp\]; st\[sp++\] = a \/ b;/case OR_DIV: a = st[--sp]; b = st[--sp]; st[sp++] = a \/ b;/'
's/st\[sp++\] = chk(a \* ((int64_t)1 << arg\[i\]))/st[sp++] = chk(a * ((int64_t)2 << arg[i]))/'
's/case OR_MIN: b = st\[--sp\]; a = st\[--sp\]; st\[sp++\] = a < b ? a : b; break;/case OR_MIN: b = st[--sp]; a = st[--sp]; st[sp++] = a > b ? a : b; break;/'
's/case OR_NEG: a = st\[--sp\]; st\[sp++\] = -a; break;/case OR_NEG: break;/'
's/case OR_CONST: st\[sp++\] = (int64_t)imm\[i\]; break;/case OR_CONST: st[sp++] = (int64_t)floor(imm[i]); break;/'
)
fail=0
for m in "${muts[@]}"; do
  cp /tmp/kf_oracle.c.orig oracle/kf_oracle.c
  sed -i "$m" oracle/kf_oracle.c
  if cmp -s oracle/kf_oracle.c /tmp/kf_oracle.c.orig; then echo "NOT APPLIED: $m"; fail=1; continue; fi
  rm -f oracle/liboracle.so
  r=$(timeout 300 python -m pytest tests/test_oracle_opcodes.py -q -p no:cacheprovider 2>&1 | tail -1)
  case "$r" in *failed*) echo "caught  : $m => $r";; *) echo "SURVIVED: $m => $r"; fail=1;; esac
done
exit $fail
