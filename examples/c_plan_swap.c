/* The activation-swap planner from plain C (include/ratel_plan.h): PAPER.md
 * §IV-D Algorithm 1 on the worked example of tests/test_swap_planner_pins.py.
 *
 *   THP_G 100 FLOP/s, BW_G 10 B/s, BW_S2M 20, BW_M2S 10, MEM_M^avail 30 B,
 *   P = 5, FLOP_f = 600; layers (A, FLOP) = (20,100) (10,300) (40,200) (30,0)
 *   -> OB order 1,0,2,3; swap {1,0,2}: A_G2M 70 B, FLOP_r 0, T_iter 19.5 s.
 *
 * Build: gcc c_plan_swap.c -I include -L <pkg> -lratel -Wl,-rpath,<pkg>
 * Host code only: no GPU and no ratel_init needed. */
#include <stdio.h>

#include "ratel.h"
#include "ratel_plan.h"

int main(void) {
  const ratel_swap_model m = {100.0, 10.0, 20.0, 10.0, 30.0, 5.0, 600.0};
  const ratel_swap_layer layers[4] = {{20, 100}, {10, 300}, {40, 200}, {30, 0}};
  int order[4];
  ratel_swap_plan plan;
  int rc = ratel_plan_activation_swap(layers, 4, &m, 0.0, order, &plan);
  if (rc != RATEL_OK) {
    printf("error %d: %s\n", rc, ratel_last_error());
    return 1;
  }
  printf("order=%d,%d,%d,%d n_swap=%d a_g2m=%g flop_r=%g t_f=%g t_b=%g t_iter=%g\n", order[0], order[1], order[2],
         order[3], plan.n_swap, plan.a_g2m, plan.flop_r, plan.t_f, plan.t_b, plan.t_iter);
  /* a bad argument is reported, not thrown */
  const ratel_swap_layer bad[1] = {{0.0, 1.0}};
  rc = ratel_plan_activation_swap(bad, 1, &m, 0.0, order, &plan);
  printf("bad_layer_rc=%d msg=%s\n", rc, ratel_last_error());
  return 0;
}
