#!/bin/bash
# Worksheet for tests/golden/jenkins32.json: Robert Jenkins' 32-bit integer
# hash, "6 shifts" variant (§VI.C l.219, ref. [17]), worked one line
# of the published listing at a time with bash's 64-bit integer arithmetic,
# every intermediate reduced mod 2^32.  It shares nothing with oracle/ (no
# C code, no import); its output was pasted into the JSON fixture once.
#   a = (a+0x7ed55d16) + (a<<12);
#   a = (a^0xc761c23c) ^ (a>>19);
#   a = (a+0x165667b1) + (a<<5);
#   a = (a+0xd3a2646c) ^ (a<<9);
#   a = (a+0xfd7046c5) + (a<<3);
#   a = (a^0xb55a4f09) ^ (a>>16);
M=0xFFFFFFFF
for x in 0 1 2 255 65536 305419896 3735928559 4294967295; do
  a=$x
  s1=$(( ((a + 0x7ed55d16) + (a << 12)) & M )); a=$s1
  s2=$(( ((a ^ 0xc761c23c) ^ (a >> 19)) & M )); a=$s2
  s3=$(( ((a + 0x165667b1) + (a << 5)) & M ));  a=$s3
  s4=$(( ((a + 0xd3a2646c) ^ (a << 9)) & M ));  a=$s4
  s5=$(( ((a + 0xfd7046c5) + (a << 3)) & M ));  a=$s5
  s6=$(( ((a ^ 0xb55a4f09) ^ (a >> 16)) & M )); a=$s6
  printf '{"in": "0x%08x", "steps": ["0x%08x", "0x%08x", "0x%08x", "0x%08x", "0x%08x", "0x%08x"]}\n' \
    $x $s1 $s2 $s3 $s4 $s5 $s6
done
