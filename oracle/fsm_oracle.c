/* fsm_oracle.c -- TEST INFRASTRUCTURE ONLY.  The plain sequential FSM loop (Fig. 1c,
 * PAPER.md:25) used as the parity oracle.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this.  It shares no code with the CUDA path.
 *
 * Definition (DFA tuple PAPER.md:61; transition step PAPER.md:213, Alg. 3 l.9):
 *   q_0 = start;  q_i = delta(q_{i-1}, x_i)  for i = 1..L
 *   result = (q_L, |{ i in [1, L] : q_i in F }|)            (reading A4: the empty prefix is
 *                                                            not counted)
 * table is state-major: delta(s, c) = table[s * alphabet + c]  (reading A3).
 * bit_mode: symbol i = bit (7 - i % 8) of byte i / 8 (MSB-first, reading A13); len counts bits.
 * A symbol >= alphabet returns ORACLE_ESYMBOL (-4) (reading A14).
 */
#include <stdint.h>

#define ORACLE_OK 0
#define ORACLE_ESYMBOL (-4)

int oracle_run(const uint32_t *table, uint32_t alphabet, uint32_t start, const uint8_t *accept,
               const uint8_t *input, uint64_t len, int bit_mode,
               uint32_t *final_state, uint64_t *accept_count)
{
    uint32_t q = start;
    uint64_t cnt = 0;
    for (uint64_t i = 0; i < len; i++) {
        uint32_t c = bit_mode ? (uint32_t)((input[i >> 3] >> (7 - (i & 7))) & 1u) : input[i];
        if (c >= alphabet)
            return ORACLE_ESYMBOL;
        q = table[(uint64_t)q * alphabet + c];
        if (accept && accept[q])
            cnt++;
    }
    *final_state = q;
    *accept_count = cnt;
    return ORACLE_OK;
}
